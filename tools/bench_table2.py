#!/usr/bin/env python
"""NEXT-2: the paper's Table II grid (Q0.2 / Q0.4 / Q1.7 / Q1.15 x truncation / nearest / stochastic
rounding x deterministic / stochastic STDP = 24 networks) trained as ONE ensemble launch per call on the
per-step engine (16-bit codes included, reading R27), MNIST-shaped synthetic images, T = 350.  Prints one JSON
line with the aggregate training throughput.  (Accuracy needs the real datasets: out of scope.)"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synthdata  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n-exc", type=int, default=400)
    ap.add_argument("--images", type=int, default=8)
    ap.add_argument("--steps", type=int, default=2)
    ap.add_argument("--T", type=int, default=350)
    a = ap.parse_args()
    import torch
    import paper_conf_date_shelm19_b200 as P
    torch.cuda.set_device(0)
    rows = {2: "2b", 4: "4b", 8: "8b", 16: "16b"}
    nets, imgs, seeds, names = [], [], [], []
    k = 0
    for bits, frac in ((2, 2), (4, 4), (8, 7), (16, 15)):             # Q0.2, Q0.4, Q1.7, Q1.15 labels (R9)
        for rounding in (0, 1, 2):
            for stdp in (1, 0):
                prm = P.preset(rows[bits], stdp_mode=stdp, rounding=rounding, frac_bits=frac, cluster_size=4,
                               engine=1, init_seed=1 + k)
                nets.append(P.Network(784, a.n_exc, bits, prm))
                n = a.images * (a.steps + 1)
                imgs.append(torch.from_numpy(synthdata.images(n, "mnist", start=1000 * k)).cuda())
                seeds.append(torch.from_numpy(synthdata.seeds(n, base_seed=400 + k).view("int64")).cuda())
                names.append(f"Q{bits}/{['trunc', 'nearest', 'stoch'][rounding]}/{['stoch', 'det'][stdp]}")
                k += 1
    sl = lambda s: slice(s * a.images, (s + 1) * a.images)  # noqa: E731
    P.present_many(nets, [x[sl(0)] for x in imgs], a.T, [x[sl(0)] for x in seeds])
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for s in range(1, a.steps + 1):
        P.present_many(nets, [x[sl(s)] for x in imgs], a.T, [x[sl(s)] for x in seeds])
    torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    n_img = len(nets) * a.images * a.steps
    print(json.dumps({"metric": "Table II grid: 24 networks trained in one ensemble launch", "value": n_img / dt,
                      "unit": "images/s", "networks": len(nets), "n_exc": a.n_exc, "T": a.T,
                      "images_per_net_per_call": a.images, "engine": "per-step (SNN_ENGINE_STEP)",
                      "cluster_size": nets[0].info()["cluster_size"], "timing": "host wall clock, synchronous calls",
                      "grid": names}))


if __name__ == "__main__":
    main()
