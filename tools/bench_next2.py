#!/usr/bin/env python
"""NEXT-2 throughput on one GPU: 16-bit codes (R27) and binary32 conductances (R28) on the per-step engine, at
the C2 network (784 -> 400, one cluster) and the C4 network (784 -> 6400, column-sharded over 4 / 7 clusters, one
snn_present_many launch).  Per config: B images per launch (learning on, T steps), W warm-up launches, K timed
launches with CUDA events on the launching stream, images/s and microseconds per simulated step.  The oracle
presents one image of the same config on one pinned core beside it.  One JSON line per config.
Usage: python tools/bench_next2.py [--only C4-16] [--no-oracle]"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synthdata  # noqa: E402

CONFIGS = [
    # name, n_exc, bits, world, preset, overrides, data, T, images per launch
    ("C2-16", 400, 16, 1, "16b", {"rounding": 2}, "mnist", 350, 8),
    ("C2-32", 400, 32, 1, "16b", {}, "mnist", 350, 8),
    ("C4-16", 6400, 16, 4, "16b", {"rounding": 2}, "fashion", 350, 4),
    ("C4-32", 6400, 32, 7, "16b", {}, "fashion", 350, 4),
]


def oracle_rate(n_exc, bits, preset, ov, kind, T):
    from oracle import oracle as O
    cpus = sorted(os.sched_getaffinity(0))
    old = set(cpus)
    os.sched_setaffinity(0, {cpus[0]})
    try:
        net = O.OracleNet(784, n_exc, bits, O.params(preset, init_seed=1, **ov))
        img, sd = synthdata.images(1, kind, start=7000)[0], int(synthdata.seeds(1, 9)[0])
        t0 = time.perf_counter()
        net.present(img, T, sd)
        return 1.0 / (time.perf_counter() - t0)
    finally:
        os.sched_setaffinity(0, old)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=1)
    ap.add_argument("--only", default="")
    ap.add_argument("--no-oracle", action="store_true")
    a = ap.parse_args()
    import torch
    import paper_conf_date_shelm19_b200 as P
    from oracle import oracle as O
    torch.cuda.set_device(0)
    for name, n_exc, bits, world, preset, ov, kind, T, B in CONFIGS:
        if a.only and name not in a.only.split(","):
            continue
        p = P.params_from_dict(O.params(preset, init_seed=1, **ov), engine=1)
        if world == 1:
            nets = [P.Network(784, n_exc, bits, p)]
        else:
            nets = [P.Network(784, n_exc, bits, p, shard=(r, world)) for r in range(world)]
            P.link_shards(nets)
        imgs = synthdata.images(B * (a.warmup + a.steps), kind, start=100)
        seeds = synthdata.seeds(B * (a.warmup + a.steps), 3)
        times = []
        for it in range(a.warmup + a.steps):
            x = np.ascontiguousarray(imgs[it * B:(it + 1) * B])
            s = np.ascontiguousarray(seeds[it * B:(it + 1) * B])
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            if world == 1:
                nets[0].present_batch(x, T, s)
                nets[0].synchronize()
            else:
                P.present_many(nets, [x] * world, T, [s] * world)   # synchronous
            t1 = time.perf_counter()
            if it >= a.warmup:
                times.append(t1 - t0)
        ts = sum(times)
        n_img = B * a.steps
        inf = nets[0].info()
        line = {"config": name, "n_exc": n_exc, "bits": bits, "world": world, "T": T, "images_per_launch": B,
                "images_per_s": n_img / ts, "us_per_step": 1e6 * ts / (n_img * T),
                "cluster_size": inf["cluster_size"], "ctas": inf["cluster_size"] * world,
                "timing": "host wall clock around synchronous launches (inputs already staged)"}
        if not a.no_oracle:
            orate = oracle_rate(n_exc, bits, preset, ov, kind, T)
            line["oracle_images_per_s_one_core"] = orate
        print(json.dumps(line), flush=True)
        for n in nets:
            n.close()


if __name__ == "__main__":
    main()
