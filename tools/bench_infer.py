#!/usr/bin/env python
"""NEXT-1 inference throughput (frozen weights): C4 network 784 -> 6400, 2-bit, fashion-shaped,
T = 350, images resident in HBM, CUDA events on the launching stream.  Prints one JSON line."""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synthdata  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--images", type=int, default=4096)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--n-exc", type=int, default=6400)
    ap.add_argument("--bits", type=int, default=2)
    ap.add_argument("--T", type=int, default=350)
    ap.add_argument("--membrane", type=int, default=0)
    ap.add_argument("--kind", default="fashion")
    a = ap.parse_args()
    import torch
    import paper_conf_date_shelm19_b200 as P
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    net = P.Network(784, a.n_exc, a.bits, P.preset({2: "2b", 4: "4b", 8: "8b"}[a.bits], membrane_mode=a.membrane))
    net.set_stream(stream.cuda_stream)
    imgs = torch.from_numpy(synthdata.images(a.images, a.kind, start=20000)).cuda()
    seeds = torch.from_numpy(synthdata.seeds(a.images, base_seed=7).view(np.int64)).cuda()
    counts = torch.zeros((a.images, a.n_exc), dtype=torch.int32, device="cuda")
    for _ in range(a.warmup):
        net.infer(imgs, a.T, seeds, counts, flags=P.SNN_ASYNC)
    torch.cuda.synchronize()
    st0 = net.infer_stats().copy()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(a.steps)]
    for e0, e1 in ev:
        e0.record(stream)
        net.infer(imgs, a.T, seeds, counts, flags=P.SNN_ASYNC)
        e1.record(stream)
    torch.cuda.synchronize()
    ms = [e0.elapsed_time(e1) for e0, e1 in ev]
    st = net.infer_stats() - st0
    t = sum(ms) / 1e3
    n = a.images * a.steps
    print(json.dumps({"metric": "inference images/s (frozen weights)", "value": n / t, "unit": "images/s",
                      "ms_per_call": sum(ms) / len(ms), "images_per_call": a.images,
                      "synaptic_events_per_s": float(st[0]) * a.n_exc / t, "act_per_step": float(st[0]) / (n * a.T),
                      "post_spikes_per_image": float(st[1]) / n, "n_exc": a.n_exc, "bits": a.bits, "T": a.T,
                      "membrane": a.membrane, "info": net.info()}))


if __name__ == "__main__":
    main()
