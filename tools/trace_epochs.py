#!/usr/bin/env python
"""Per-epoch phase breakdown of the event engine from the %globaltimer trace (snn_set_trace).
Usage: python tools/trace_epochs.py [--n-exc 6400 --bits 2 --images 4 --cluster-size 0]"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synthdata  # noqa: E402
import paper_conf_date_shelm19_b200 as P  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n-exc", type=int, default=6400)
    ap.add_argument("--bits", type=int, default=2)
    ap.add_argument("--images", type=int, default=4)
    ap.add_argument("--T", type=int, default=350)
    ap.add_argument("--cluster-size", type=int, default=0)
    ap.add_argument("--kind", default="fashion")
    ap.add_argument("--gamma-pot", type=float, default=None)
    ap.add_argument("--gamma-dep", type=float, default=None)
    ap.add_argument("--membrane", type=int, default=0)
    a = ap.parse_args()
    pre = {2: "2b", 4: "4b", 8: "8b"}[a.bits]
    prm = P.preset(pre, cluster_size=a.cluster_size, membrane_mode=a.membrane)
    if a.gamma_pot is not None:
        prm.gamma_pot = a.gamma_pot
    if a.gamma_dep is not None:
        prm.gamma_dep = a.gamma_dep
    net = P.Network(784, a.n_exc, a.bits, prm)
    print("info", net.info())
    imgs = synthdata.images(a.images + 2, a.kind)
    seeds = synthdata.seeds(a.images + 2, 1)
    net.present_batch(imgs[:2], a.T, seeds[:2])            # warm-up
    net.set_trace(64 * a.images)
    net.reset_stats()
    net.present_batch(imgs[2:], a.T, seeds[2:])
    tr = net.trace().astype(np.int64)                       # (cs, E, 8)
    prof = tr[:, -1, :].copy()
    print("prof raw", prof[:2].tolist())
    tr = tr[:, :-1, :]
    for r in range(prof.shape[0]):
        if (prof[r, 0] >> 32) & 0xFFFFFFFF == 0xFFFFFFFF and prof[r, 4] > 0:
            nbk = prof[r, 4]
            print(f"CTA {r} slowest warp {prof[r,0] & 0xFFFF} cycles/step: integrate {prof[r,1]/nbk:.0f}  ltd {prof[r,2]/nbk:.0f}  seq {prof[r,3]/nbk:.0f}"
                  f" (of which LTD events {prof[r,6]/nbk:.0f}, {((prof[r,0] >> 16) & 0xFFFF)/nbk:.2f} events/step)  whole-loop {prof[r,5]/nbk:.0f}  (block steps {nbk})")
    st = net.stats()
    cs, E, _ = tr.shape
    valid = tr[0, :, 7] > 0
    tr = tr[:, valid]
    E = tr.shape[1]
    k0 = tr[0, :, 0] & 0xFFFFFFFF
    kind = tr[0, :, 1] >> 32
    Pst = tr[0, :, 1] & 0xFFFFFFFF
    start = tr[:, :, 2].min(axis=0)
    spec_end = tr[:, :, 3]
    summ = tr[:, :, 4]
    exch = tr[:, :, 5]
    depth = tr[:, :, 6] & 0xFFFF
    late = tr[:, :, 6] >> 16                                 # longest warp loop of the CTA (cycles)
    comm = tr[:, :, 7]
    end = tr[:, :, 7]
    tot = end.max(axis=0) - start
    spec = spec_end.max(axis=0) - start
    spread = spec_end.max(axis=0) - spec_end.min(axis=0)
    wait = exch.max(axis=0) - summ.max(axis=0)
    commit = comm.max(axis=0) - exch.min(axis=0)
    ltp = end.max(axis=0) - comm.min(axis=0)
    adv = np.diff(np.append(k0, k0[-1]))
    print("stats", [int(x) for x in st[:13]])
    print(f"cluster {cs}  epochs {E}  images {a.images}  epochs/image {E / a.images:.1f}  post spikes {int(st[1])}")
    print(f"per-epoch mean ns: total {tot.mean():.0f}  speculation {spec.mean():.0f} (spread across CTAs {spread.mean():.0f})"
          f"  summary->exchanged {wait.mean():.0f}  commit {commit.mean():.0f}  LTP+tail {ltp.mean():.0f}")
    print(f"per-image us: {tot.sum() / a.images / 1e3:.1f}   sum of per-epoch speculation {spec.sum() / a.images / 1e3:.1f}")
    print(f"steps per epoch (mean) {np.mean(adv[adv > 0]):.1f}; speculation ns/step {spec.sum() / max(1, a.T * a.images):.0f}")
    own = spec_end - tr[:, :, 2]                         # per-CTA speculation duration
    skew = tr[:, :, 2] - start[None, :]                    # per-CTA start skew
    steps = (Pst - k0 + 1).astype(float)
    print(f"per-CTA speculation ns: mean {own.mean():.0f}  max-over-CTAs mean {own.max(axis=0).mean():.0f}  "
          f"-> {own.max(axis=0).sum() / steps.sum():.0f} ns/step (max CTA)  {own.mean(axis=0).sum() / steps.sum():.0f} ns/step (mean CTA)")
    print(f"start skew ns: mean {skew.mean():.0f}  max {skew.max(axis=0).mean():.0f}")
    rate = own / np.maximum(1, depth)                       # ns per speculated step, per CTA per epoch
    crit = own.argmax(axis=0)
    print(f"critical CTA: ns/step {np.mean([rate[crit[e], e] for e in range(E)]):.0f} at depth "
          f"{np.mean([depth[crit[e], e] for e in range(E)]):.1f};  other CTAs ns/step {np.median(rate):.0f} at depth {np.median(depth):.1f}")
    bw = tr[:, :, 4]
    parts = np.array([[(bw[crit[e], e] >> (16 * k)) & 0xFFFF for k in range(4)] for e in range(E)]) * 16.0
    dc = np.array([max(1, depth[crit[e], e]) for e in range(E)])
    print("critical CTA slowest warp cycles/step: integrate %.0f  ltd-draws %.0f  seq %.0f (LTD events %.0f)" %
          tuple((parts / dc[:, None]).mean(axis=0)))
    print(f"longest warp loop: critical CTA {np.mean([late[crit[e], e] for e in range(E)]) / 1.965:.0f} ns "
          f"(= {np.mean([late[crit[e], e] / max(1, depth[crit[e], e]) for e in range(E)]):.0f} cycles/step), median CTA {np.median(late) / 1.965:.0f} ns")
    print("first 12 epochs: k0 P kind | spec(ns) spread wait commit ltp")
    for e in range(min(12, E)):
        print(f"{k0[e]:4d} {Pst[e]:5d} {kind[e]} | {spec[e]:7d} {spread[e]:6d} {wait[e]:6d} {commit[e]:6d} {ltp[e]:6d}")


if __name__ == "__main__":
    main()
