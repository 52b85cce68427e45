#!/usr/bin/env python
"""(Cycle split columns need the library built with -DSNN_LEAN_TRACE_CYCLES=1.)  Per-CTA speculation time of the lean event kernel (snn_set_trace records), split by the CTA's role in
the epoch: the CTA that held the previous winner (LTP at the epoch start, LTD-active column), the CTA
holding this epoch's winner, and the others.  Usage: python tools/trace_lean.py [--images 8]"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synthdata  # noqa: E402
import paper_conf_date_shelm19_b200 as P  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--images", type=int, default=8)
a = ap.parse_args()
net = P.Network(784, 6400, 2, P.preset("2b"))
imgs = synthdata.images(a.images + 2, "fashion")
seeds = synthdata.seeds(a.images + 2, 1)
net.present_batch(imgs[:2], 350, seeds[:2])
net.set_trace(64 * a.images)
net.present_batch(imgs[2:], 350, seeds[2:])
tr = net.trace().astype(np.int64)
cs = tr.shape[0]
valid = tr[0, :, 7] > 0
tr = tr[:, valid]
E = tr.shape[1]
cols = 6400 // cs
start, end_spec, exch, end = tr[:, :, 2], tr[:, :, 3], tr[:, :, 5], tr[:, :, 7]
nblk, ngen, nsolo = tr[:, :, 0] >> 48, tr[:, :, 1] >> 48, tr[:, :, 4] >> 48
tr[:, :, 0] &= 0xFFFFFFFFFFFF
tr[:, :, 1] &= 0xFFFFFFFFFFFF
tr[:, :, 4] &= 0xFFFFFFFFFFFF
W = tr[0, :, 4]
k0 = tr[0, :, 0] & 0xFFFFFFFF
Pst = tr[0, :, 1] & 0xFFFFFFFF
own = end_spec - start
gstart = start.min(axis=0)
lat = end_spec - gstart[None, :]
roles = {"prev-winner CTA": [], "winner CTA": [], "other CTAs": []}
for e in range(1, E):
    wprev = W[e - 1] // cols if W[e - 1] != 0xFFFFFFFF else -1
    wcur = W[e] // cols if W[e] != 0xFFFFFFFF else -1
    for r in range(cs):
        key = "prev-winner CTA" if r == wprev else ("winner CTA" if r == wcur else "other CTAs")
        roles[key].append((own[r, e], lat[r, e], start[r, e] - gstart[e]))
for k, v in roles.items():
    v = np.array(v, dtype=np.float64)
    print(f"{k:16s} n={len(v):5d}  own spec {v[:, 0].mean():7.0f} ns  finish after global start {v[:, 1].mean():7.0f} ns"
          f"  start lag {v[:, 2].mean():6.0f} ns")
sp = tr[:, :, 6]
split = np.stack([(sp >> 48) & 0xFFFF, (sp >> 32) & 0xFFFF, (sp >> 16) & 0xFFFF, sp & 0xFFFF], -1) * 16.0
for k in roles:
    pass
pw = [W[e - 1] // cols if W[e - 1] != 0xFFFFFFFF else -1 for e in range(1, E)]
sel_p = np.array([split[pw[e - 1], e] for e in range(1, E) if pw[e - 1] >= 0])
sel_o = np.array([split[r, e] for e in range(1, E) for r in range(cs) if r != pw[e - 1]])
for name, x in (("prev-winner CTA", sel_p), ("other CTAs", sel_o)):
    print(f"{name:16s} slowest warp cycles/epoch: loop {x[:, 0].mean():7.0f}  held+solo {x[:, 1].mean():6.0f}  "
          f"block {x[:, 2].mean():6.0f}  general {x[:, 3].mean():6.0f}")
crit = lat.argmax(axis=0)
wp = np.array([W[e - 1] // cols if W[e - 1] != 0xFFFFFFFF else -1 for e in range(1, E)])
print(f"critical CTA == previous winner's CTA in {np.mean(crit[1:] == wp) * 100:.0f}% of epochs")
ev = (tr[0, :, 1] >> 32) == 1                  # epochs that ended with a post spike (P = t*)
steps = (Pst[ev] - k0[ev] + 1).astype(float)
print(f"epochs {E}, steps/epoch {steps.mean():.1f}, per-epoch: spec (global) {lat.max(axis=0).mean():.0f} ns, "
      f"exchange->end {(end.max(axis=0) - exch.min(axis=0)).mean():.0f} ns, total {(end.max(axis=0) - gstart).mean():.0f} ns")
ph = tr[:, :, 6]
win = [(e, W[e] // cols) for e in range(E) if W[e] != 0xFFFFFFFF]     # the winner's CTA runs the phases
if win:
    x = np.array([[(ph[r, e] >> (48 - 16 * q)) & 0xFFFF for q in range(4)] for e, r in win], dtype=np.float64) * 8
    x = x[x.sum(axis=1) > 0]
    if len(x):
        print(f"winner CTA after the exchange (cycles, phase-stamp build): draw {x[:, 0].mean():.0f}, LTP {x[:, 1].mean():.0f}, "
              f"barrier {x[:, 2].mean():.0f}, sums {x[:, 3].mean():.0f}")
print(f"warp-steps per CTA per epoch: block {nblk.mean():.1f}  general {ngen.mean():.1f}  solo {nsolo.mean():.1f}")
