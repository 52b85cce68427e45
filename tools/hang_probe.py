"""Debug helper: run one presentation config in a subprocess with a timeout, for growing T."""
import os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import sys, numpy as np
sys.path.insert(0, %r)
import synthdata, paper_conf_date_shelm19_b200 as P
from oracle import oracle as O
T = int(sys.argv[1]); eng = int(sys.argv[2]); nimg = int(sys.argv[3])
p = O.params("2b", f_min_hz=200.0, f_max_hz=1000.0, gamma_dep=1.0, tau_dep=50.0, v_spike=0.5, membrane_mode=1, init_seed=13)
g = P.Network(784, 256, 2, P.params_from_dict(p, engine=eng))
o = O.OracleNet(784, 256, 2, p)
import time
for img, sd in zip(synthdata.images(nimg, "fashion", start=3), synthdata.seeds(nimg, 13)):
    t0 = time.time(); g.present(img, T, int(sd)); t1 = time.time(); o.present(img, T, int(sd)); t2 = time.time()
    print("gpu s", round(t1 - t0, 3), "oracle s", round(t2 - t1, 3), flush=True)
    print("T", T, "stats", g.stats()[:13].tolist(), "eq", np.array_equal(g.weights(), o.weights()), np.array_equal(g.spikes(), o.spikes()), flush=True)
''' % ROOT
for T in [int(x) for x in sys.argv[1].split(",")]:
    for eng in (0,):
        try:
            r = subprocess.run([sys.executable, "-c", CHILD, str(T), str(eng), sys.argv[2] if len(sys.argv) > 2 else "1"],
                               capture_output=True, text=True, timeout=40)
            print(r.stdout.strip(), r.stderr.strip()[-300:], flush=True)
        except subprocess.TimeoutExpired as e:
            print("T", T, "TIMEOUT", (e.stdout or b"")[-300:], flush=True)
