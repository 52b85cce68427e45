#!/usr/bin/env python
"""C5 measurement: an ensemble of independent 784 -> 400 networks (bit widths {2,4,8}[k mod 3], each with its
Table I row, seed k) presented together with snn_present_many (one launch per bit width, all clusters
co-resident), MNIST-shaped images, T = 350.  One GPU holds one group of --nets networks (SURVEY §8(d) C5:
8 per GPU x 8 GPUs).  Prints one JSON line: aggregate training images/s."""
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
    ap.add_argument("--nets", type=int, default=8)
    ap.add_argument("--images", type=int, default=16)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--T", type=int, default=350)
    a = ap.parse_args()
    import torch
    import paper_conf_date_shelm19_b200 as P
    torch.cuda.set_device(0)
    nets, imgs, seeds = [], [], []
    for k in range(a.nets):
        bits = (2, 4, 8)[k % 3]
        nets.append(P.Network(784, 400, bits, P.preset({2: "2b", 4: "4b", 8: "8b"}[bits], init_seed=1 + k,
                                                       cluster_size=2)))
        imgs.append(torch.from_numpy(synthdata.images(a.images * (a.steps + 1), "mnist", start=10000 * k)).cuda())
        seeds.append(torch.from_numpy(synthdata.seeds(a.images * (a.steps + 1), base_seed=200 + k).view("int64")).cuda())
    sl = lambda s: slice(s * a.images, (s + 1) * a.images)  # noqa: E731
    P.present_many(nets, [x[sl(0)] for x in imgs], a.T, [x[sl(0)] for x in seeds])     # warm-up
    for n in nets:
        n.reset_stats()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for s in range(1, a.steps + 1):
        P.present_many(nets, [x[sl(s)] for x in imgs], a.T, [x[sl(s)] for x in seeds])
    torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    n_img = a.nets * a.images * a.steps
    act = sum(int(n.stats()[0]) for n in nets)
    print(json.dumps({"metric": "C5 ensemble training images/s (784->400, bits {2,4,8})", "value": n_img / dt,
                      "unit": "images/s", "nets": a.nets, "images_per_net_per_call": a.images, "T": a.T,
                      "per_net_images_per_s": n_img / dt / a.nets, "synaptic_events_per_s": act * 400 / dt,
                      "timing": "host wall clock around synchronous snn_present_many calls",
                      "cluster_size": nets[0].info()["cluster_size"]}))


if __name__ == "__main__":
    main()
