#!/usr/bin/env python
"""Throughput of every SURVEY §8(d) config on one GPU, next to the CPU oracle.

Per config: a batch of B images per snn_present_batch launch, W warm-up launches, K timed launches (CUDA
events on the launching stream around each launch, L2 flushed between launches), the presentation kernel's
own time from the library's events (snn_set_profile), and -- lean kernel only -- the latency floor
(SNN_FLOOR_PROBE).  The oracle presents a few images of the same config on one pinned core.  One JSON line
per config."""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synthdata  # noqa: E402

SMEM_PEAK_GBS = 128 * 148 * 1965e6 / 1e9     # derived SMEM crossbar peak (B300_MICROARCH 128 B/clk/SM)

CONFIGS = [
    # name, n_exc, bits, preset, overrides, data, T, images per launch, oracle images
    ("C1", 100, 8, "8b", {}, "mnist", 100, 20, 20),
    ("C2-S", 400, 8, "8b", {"wta_mode": 1}, "mnist", 350, 32, 3),
    ("C2-D", 400, 8, "8b", {"wta_mode": 1, "stdp_mode": 1, "rounding": 1}, "mnist", 350, 32, 3),
    ("C3-1-22", 1600, 2, "2b", {}, "mnist", 350, 32, 2),
    ("C3-5-78", 1600, 2, "2b", {"f_min_hz": 5.0, "f_max_hz": 78.0}, "mnist", 100, 32, 3),
    ("C3-5-156", 1600, 2, "2b", {"f_min_hz": 5.0, "f_max_hz": 156.0}, "mnist", 100, 32, 3),
    ("C3-10-312", 1600, 2, "2b", {"f_min_hz": 10.0, "f_max_hz": 312.0}, "mnist", 100, 32, 3),
    ("C4", 6400, 2, "2b", {}, "fashion", 350, 32, 1),
    ("C4-HF", 6400, 2, "hf", {}, "fashion", 100, 32, 2),
]


def oracle_rate(n_exc, bits, preset, ov, kind, T, n):
    from oracle import oracle as O
    cpus = sorted(os.sched_getaffinity(0))
    old = set(cpus)
    os.sched_setaffinity(0, {cpus[0]})
    try:
        net = O.OracleNet(784, n_exc, bits, O.params(preset, init_seed=1, **ov))
        imgs, seeds = synthdata.images(n, kind, start=7000), synthdata.seeds(n, 9)
        t0 = time.perf_counter()
        for x, s in zip(imgs, seeds):
            net.present(x, T, int(s))
        return n / (time.perf_counter() - t0)
    finally:
        os.sched_setaffinity(0, old)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--only", default="")
    ap.add_argument("--no-oracle", action="store_true")
    a = ap.parse_args()
    import torch
    import paper_conf_date_shelm19_b200 as P
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device="cuda")
    for name, n_exc, bits, preset, ov, kind, T, B, n_or in CONFIGS:
        if a.only and name not in a.only.split(","):
            continue
        net = P.Network(784, n_exc, bits, P.preset(preset, init_seed=1, **ov))
        net.set_stream(stream.cuda_stream)
        tot = B * (a.warmup + a.steps)
        imgs = torch.from_numpy(synthdata.images(tot, kind)).cuda()
        seeds = torch.from_numpy(synthdata.seeds(tot, 1).view(np.int64)).cuda()
        sl = lambda k: slice(k * B, (k + 1) * B)  # noqa: E731
        for k in range(a.warmup):
            net.present_batch(imgs[sl(k)], T, seeds[sl(k)], None, flags=P.SNN_ASYNC)
        torch.cuda.synchronize()
        net.reset_stats()
        net.set_profile(True)
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(a.steps)]
        for i in range(a.steps):
            flush.fill_(i & 0xFF)
            ev[i][0].record(stream)
            net.present_batch(imgs[sl(a.warmup + i)], T, seeds[sl(a.warmup + i)], None, flags=P.SNN_ASYNC)
            ev[i][1].record(stream)
        torch.cuda.synchronize()
        kms, kn = net.profile()
        net.set_profile(False)
        step_s = sum(x.elapsed_time(y) for x, y in ev) / 1e3
        st = net.stats().astype(np.float64)
        images = B * a.steps
        info = net.info()
        # algorithmic SMEM bytes: integration reads + STDP trial reads + event writes
        alg = st[0] * n_exc * bits / 8 + (st[2] + st[4]) * bits / 8 + (st[3] + st[5]) * bits / 8
        line = {"config": name, "n_exc": n_exc, "bits": bits, "T": T, "data": kind, "overrides": ov,
                "kernel": "lean" if info["lean"] else ("event" if info["engine"] == 0 else "step"),
                "cluster_size": info["cluster_size"], "images_per_launch": B,
                "images_per_s": images / step_s, "synaptic_events_per_s": st[0] * n_exc / step_s,
                "kernel_share_of_step": (kms / 1e3) / step_s if kn else None,
                "smem_roofline_frac": (alg / (kms / 1e3)) / 1e9 / SMEM_PEAK_GBS if kn else None,
                "post_spikes_per_image": st[1] / images, "act_per_step": st[0] / (images * T),
                "epochs_per_image": st[8] / images}
        if info["lean"] and kn:
            net.set_profile(True)
            for i in range(2):
                net.present_batch(imgs[sl(i)], T, seeds[sl(i)], None, flags=P.SNN_ASYNC | P.snn.SNN_FLOOR_PROBE)
            fms, fn = net.profile()
            net.set_profile(False)
            line["latency_floor_frac"] = (fms / fn) / (kms / kn)
        if not a.no_oracle:
            orate = oracle_rate(n_exc, bits, preset, ov, kind, T, n_or)
            line["oracle_images_per_s_1core"] = orate
            line["speedup_vs_oracle_1core"] = line["images_per_s"] / orate
        print(json.dumps(line), flush=True)
        net.close()


if __name__ == "__main__":
    main()
