mkdir -p gpurun_out
(timeout 120 python tools/trace_epochs.py --images 8; echo ===GDEP0; timeout 120 python tools/trace_epochs.py --images 8 --gamma-dep 0; echo ===GPOT0; timeout 120 python tools/trace_epochs.py --images 8 --gamma-pot 0; echo ===GENERAL; SNN_NO_LEAN=1 timeout 120 python tools/trace_epochs.py --images 8) > gpurun_out/trace.txt 2>&1
for a in "" "--gamma-dep 0" "--gamma-pot 0"; do echo "== $a"; timeout 120 python - $a <<'PY'
import sys, time, numpy as np, torch
sys.path.insert(0, '.')
import synthdata, paper_conf_date_shelm19_b200 as P
args = sys.argv[1:]
kw = {}
if '--gamma-dep' in args: kw['gamma_dep'] = 0.0
if '--gamma-pot' in args: kw['gamma_pot'] = 0.0
net = P.Network(784, 6400, 2, P.preset('2b', **kw))
imgs = synthdata.images(40, 'fashion'); seeds = synthdata.seeds(40, 1)
net.present_batch(imgs[:8], 350, seeds[:8])
net.reset_stats()
t0 = time.perf_counter(); net.present_batch(imgs[8:], 350, seeds[8:]); dt = time.perf_counter() - t0
st = net.stats()
print(f"{32/dt:.0f} images/s  post spikes/img {st[1]/32:.1f}  epochs/img {st[8]/32:.1f}  ltd trials/img {st[2]/32:.0f} events/img {st[3]/32:.0f}  ltp trials {st[4]/32:.0f}")
PY
done >> gpurun_out/trace.txt 2>&1
cat gpurun_out/trace.txt | grep -v "^prof raw\|^info"
