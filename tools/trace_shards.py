#!/usr/bin/env python
"""Per-epoch timing of the column-sharded event engine on one GPU (K linked shards, one launch).
Usage: python tools/trace_shards.py --shards 4 [--images 4]"""
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
    ap.add_argument("--shards", type=int, default=2)
    ap.add_argument("--images", type=int, default=4)
    ap.add_argument("--n-exc", type=int, default=6400)
    a = ap.parse_args()
    K = a.shards
    prm = P.preset("2b", membrane_mode=0)
    if K > 1:
        nets = [P.Network(784, a.n_exc, 2, prm, shard=(r, K)) for r in range(K)]
        P.link_shards(nets)
    else:
        nets = [P.Network(784, a.n_exc, 2, prm)]
    print("info", nets[0].info())
    imgs = synthdata.images(a.images + 2, "fashion")
    seeds = synthdata.seeds(a.images + 2, 1)
    P.present_many(nets, [imgs[:2]] * K, 350, [seeds[:2]] * K)
    for n in nets:
        n.set_trace(64 * a.images)
    P.present_many(nets, [imgs[2:]] * K, 350, [seeds[2:]] * K)
    trs = [n.trace().astype(np.int64)[:, :-1, :] for n in nets]      # (cs, E, 8) per shard
    valid = trs[0][0, :, 7] > 0
    trs = [t[:, valid] for t in trs]
    E = trs[0].shape[1]
    t0 = min(t[:, :, 2].min() for t in trs)
    start = np.stack([t[:, :, 2].min(axis=0) for t in trs])          # (K, E)
    spec_end = np.stack([t[:, :, 3].max(axis=0) for t in trs])
    summ = np.stack([t[:, :, 4].max(axis=0) for t in trs]) if False else None
    exch = np.stack([t[:, :, 5].max(axis=0) for t in trs])
    exch_min = np.stack([t[:, :, 5].min(axis=0) for t in trs])
    end = np.stack([t[:, :, 7].max(axis=0) for t in trs])
    epoch = end.max(axis=0)[1:] - end.max(axis=0)[:-1]
    spec = spec_end - start
    print(f"epochs {E}  per-epoch (median us): whole {np.median(epoch)/1e3:.2f}")
    print("  spec duration per shard  ", [f"{np.median(spec[k])/1e3:.2f}" for k in range(K)])
    print("  max-spec over shards     ", f"{np.median(spec.max(axis=0))/1e3:.2f}")
    print("  spec_end -> exchanged    ", [f"{np.median(exch[k]-spec_end[k])/1e3:.2f}" for k in range(K)])
    print("  last spec_end(world) -> exchanged", [f"{np.median(exch[k]-spec_end.max(axis=0))/1e3:.2f}" for k in range(K)])
    print("  exchanged spread in shard", [f"{np.median(exch[k]-exch_min[k])/1e3:.2f}" for k in range(K)])
    print("  exchanged -> end (commit)", [f"{np.median(end[k]-exch[k])/1e3:.2f}" for k in range(K)])
    print("  start skew vs earliest   ", [f"{np.median(start[k]-start.min(axis=0))/1e3:.2f}" for k in range(K)])
    print("  mean whole epoch", f"{np.mean(epoch)/1e3:.2f}", "total ms", (end.max() - t0) / 1e6)


if __name__ == "__main__":
    main()
