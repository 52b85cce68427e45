#!/usr/bin/env python
"""Benchmark of the simulate-and-learn path (driver contract).

Workload (BASELINE.json metric "synaptic events/sec & training images/sec (784->6400, 2-bit)"):
config C4 -- one 784 -> 6400 LIF network, 2-bit codes, stochastic STDP (Table I "2 bit" row),
fashion-shaped synthetic images, T = 350 steps (350 ms at dt = 1 ms), 1-22 Hz, HARD WTA, fp32
membranes.  A "step" = one snn_present_batch launch presenting B images back to back (online
learning: the images of a step are sequential by construction).  value = training images/s with
inputs resident in HBM; secondary = synaptic events/s (sum_t act(t) * n_exc).

Multi-GPU (torchrun, N > 1): one independent network per GPU (replicas, "scaling": "weak"); no
data-path collective -- one network's steps are strictly sequential.

--impl reference: the CPU oracle (oracle/) as it stands, single-threaded, timed on the host.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import synthdata  # noqa: E402

METRIC = "synaptic events/sec & training images/sec (784→6400, 2-bit) at 1/2/4/8 B200"
N_IN, N_EXC, BITS, T_STEPS = 784, 6400, 2, 350
WORKLOAD = "C4: 784->6400 LIF, 2-bit codes, stochastic STDP (Table I 2-bit row), fashion-shaped synthetic, T=350, 1-22 Hz, HARD WTA, fp32 membranes"
SMEM_BYTES_PER_CLK_PER_SM = 128   # B300_MICROARCH.md "smem crossbar BW 128/N B/cyc/SM"
N_SM = 148


def _dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled DURING the timed region (B200_PROFILING.md)."""
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.path = os.path.join("/tmp", f"bench_clocks_{os.getpid()}.csv")

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "50"], stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self) -> dict:
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, smax, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in open(self.path):
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                smax = float(f[2])
            except ValueError:
                continue
            for n, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": smax,
                "reasons": sorted(reasons), "samples": len(sm)}


def run_reference(args):
    """Reference arm: the CPU oracle as it stands, single-threaded, on a bounded sample."""
    ws, rank, _ = _dist_env()
    if rank != 0:
        return
    from oracle import oracle as O
    p = O.params("2b", membrane_mode=0, init_seed=1)
    net = O.OracleNet(N_IN, N_EXC, BITS, p)
    imgs = synthdata.images(args.warmup + args.steps, "fashion")
    seeds = synthdata.seeds(args.warmup + args.steps, base_seed=1)
    per = 1  # images per reference step (bounded sample)
    for k in range(args.warmup):
        net.present(imgs[k], T_STEPS, int(seeds[k]))
    t0 = time.perf_counter()
    act = 0
    for k in range(args.warmup, args.warmup + args.steps):
        net.present(imgs[k], T_STEPS, int(seeds[k]))
        act += int(net.stats()[0])
    dt = time.perf_counter() - t0
    ips = args.steps * per / dt
    line = {
        "impl": "reference", "metric": METRIC, "value": ips, "unit": "images/s", "n_gpus": ws,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * dt / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32/u2", "data": "synthetic",
        "config": {"workload": WORKLOAD, "images_per_step": per, "n_in": N_IN, "n_exc": N_EXC, "bits": BITS,
                   "T": T_STEPS},
        "secondary": {"synaptic_events_per_s": act * N_EXC / dt},
        "cpu_baseline": {"value": ips, "unit": "images/s", "cores": 1, "kind": "oracle",
                         "sample": f"{args.steps} fashion images of C4 presented by oracle_present, single thread"},
        "e2e": {"value": ips, "unit": "images/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def cpu_baseline(n_images: int) -> dict:
    from oracle import oracle as O
    p = O.params("2b", membrane_mode=0, init_seed=1)
    net = O.OracleNet(N_IN, N_EXC, BITS, p)
    imgs = synthdata.images(n_images, "fashion", start=1000)
    seeds = synthdata.seeds(n_images, base_seed=3)
    t0 = time.perf_counter()
    for k in range(n_images):
        net.present(imgs[k], T_STEPS, int(seeds[k]))
    dt = time.perf_counter() - t0
    return {"value": n_images / dt, "unit": "images/s", "cores": 1, "kind": "oracle",
            "sample": f"{n_images} fashion images of C4 (784->6400, 2-bit, T=350) via oracle_present, 1 thread"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="b200", choices=["b200", "reference"])
    ap.add_argument("--images-per-step", type=int, default=32)
    ap.add_argument("--cluster-size", type=int, default=0)
    ap.add_argument("--membrane", type=int, default=0, help="0 fp32, 1 Q15.16")
    ap.add_argument("--cpu-images", type=int, default=10, help="oracle images for cpu_baseline (0 = skip)")
    ap.add_argument("--no-floor", action="store_true")
    ap.add_argument("--engine", type=int, default=0, help="0 event-driven epochs, 1 per-step exchange")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import paper_conf_date_shelm19_b200 as P

    ws, rank, local = _dist_env()
    ndev = torch.cuda.device_count()
    local_dev = local % max(1, ndev)
    torch.cuda.set_device(local_dev)
    dist = None
    coll_dev = torch.device("cuda", local_dev)
    if ws > 1:
        import torch.distributed as dist
        if ndev >= ws:      # one process per GPU (the driver's layout): NCCL
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_dev))
        else:               # functional check with ranks sharing a GPU: gloo on CPU tensors
            dist.init_process_group("gloo")
            coll_dev = torch.device("cpu")
    dev = torch.device("cuda", local_dev)
    # a dedicated (non-default) stream: the handle launches on it and the CUDA events are recorded on it
    stream = torch.cuda.Stream(dev)
    torch.cuda.set_stream(stream)

    B = args.images_per_step
    params = P.preset("2b", membrane_mode=args.membrane, init_seed=1 + rank, cluster_size=args.cluster_size,
                      engine=args.engine)
    net = P.Network(N_IN, N_EXC, BITS, params)
    net.set_stream(stream.cuda_stream)
    info = net.info()

    n_steps_total = args.warmup + args.steps
    pool_n = B * n_steps_total
    imgs_h = synthdata.images(pool_n, "fashion", start=rank * 100000)
    seeds_h = synthdata.seeds(pool_n, base_seed=1 + rank)
    imgs_d = torch.from_numpy(imgs_h).to(dev)
    seeds_d = torch.from_numpy(seeds_h.view(np.int64)).to(dev)
    counts_d = torch.zeros(pool_n, dtype=torch.int32, device=dev)
    flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=dev)   # > 126 MB L2

    def step(k, flags=0):
        sl = slice(k * B, (k + 1) * B)
        net.present_batch(imgs_d[sl], T_STEPS, seeds_d[sl], counts_d[sl], flags=flags | P.SNN_ASYNC)

    for k in range(args.warmup):
        step(k)
    torch.cuda.synchronize()
    net.reset_stats()
    launches0 = net.info()["launches"]

    # ---- timed region: device time per step (CUDA events on the launching stream), L2 flushed between steps
    sampler = ClockSampler(local)
    sampler.start()
    time.sleep(0.15)
    if dist:
        dist.barrier()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    for i in range(args.steps):
        flush.random_(0, 255) if i == 0 else flush.fill_(i & 0xFF)
        ev[i][0].record(stream)
        step(args.warmup + i)
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    if dist:
        dist.barrier()
    clocks = sampler.stop()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    dev_s = sum(step_ms) / 1e3
    stats = net.stats()
    launches = net.info()["launches"] - launches0
    images = B * args.steps
    events = int(stats[0]) * N_EXC
    # max over ranks of the device time
    if dist:
        t = torch.tensor([dev_s], device=coll_dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dev_s = float(t.item())
        tot = torch.tensor([images, events], device=coll_dev, dtype=torch.float64)
        dist.all_reduce(tot, op=dist.ReduceOp.SUM)
        images, events = int(tot[0].item()), int(tot[1].item())
    value = images / dev_s
    ev_rate = events / dev_s

    # ---- latency floor.  Event engine: the path needs one cluster exchange per epoch (post spike), so
    # its synchronisation floor is epochs x the measured barrier.cluster cost at this cluster size
    # (profiles/r01_sync_probe.txt, 128 threads); per-step engine: measured live with SNN_FLOOR_PROBE.
    floor = None
    if args.engine == 0:
        probe_ns = {1: 380.7, 2: 444.0, 4: 485.5, 8: 572.6, 16: 760.9}
        cs = info["cluster_size"]
        key = min(probe_ns, key=lambda k: abs(k - cs))
        per_image_us = 1e3 * (sum(step_ms) / args.steps) / B
        ep = int(stats[8]) / (B * args.steps)
        floor = {"kind": "event engine: epochs x cluster-exchange cost",
                 "epochs_per_image": ep, "exchange_ns": probe_ns[key],
                 "t_floor_us_per_image": ep * probe_ns[key] / 1e3, "t_image_us": per_image_us,
                 "frac": ep * probe_ns[key] / 1e3 / per_image_us}
    if not args.no_floor and args.engine == 1:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        step(args.warmup, flags=P.snn.SNN_FLOOR_PROBE)
        e1.record(stream)
        torch.cuda.synchronize()
        floor_ms = e0.elapsed_time(e1)
        floor = {"t_floor_us_per_step": 1e3 * floor_ms / (B * T_STEPS),
                 "t_step_us": 1e3 * (sum(step_ms) / args.steps) / (B * T_STEPS)}
        floor["frac"] = floor["t_floor_us_per_step"] / floor["t_step_us"]

    # ---- e2e: the public API with HOST buffers (pinned), H2D of inputs + D2H of the per-image result
    imgs_pin = torch.from_numpy(imgs_h).pin_memory()
    seeds_pin = torch.from_numpy(seeds_h.view(np.int64)).pin_memory()
    counts_pin = torch.zeros(pool_n, dtype=torch.int32).pin_memory()
    net2_params = P.preset("2b", membrane_mode=args.membrane, init_seed=1 + rank, cluster_size=args.cluster_size,
                      engine=args.engine)
    net2 = P.Network(N_IN, N_EXC, BITS, net2_params)
    net2.set_stream(stream.cuda_stream)
    for k in range(args.warmup):
        sl = slice(k * B, (k + 1) * B)
        net2.present_batch(imgs_pin[sl], T_STEPS, seeds_pin[sl], counts_pin[sl])
    if dist:
        dist.barrier()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for i in range(args.steps):
        k = args.warmup + i
        sl = slice(k * B, (k + 1) * B)
        net2.present_batch(imgs_pin[sl], T_STEPS, seeds_pin[sl], counts_pin[sl])   # synchronous: result on host
    torch.cuda.synchronize()
    e2e_s = time.perf_counter() - t0
    if dist:
        t = torch.tensor([e2e_s], device=coll_dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_s = float(t.item())
    e2e = {"value": images / e2e_s, "unit": "images/s", "h2d_bytes_per_step": B * (N_IN + 8),
           "d2h_bytes_per_step": B * 4, "timing": "host wall clock around synchronous snn_present_batch calls"}

    # ---- roofline of the dominant kernel (present_kernel; one launch per step)
    bits_b = BITS / 8.0
    alg_bytes = (int(stats[0]) * N_EXC * bits_b                       # integration reads (a2)
                 + (int(stats[2]) + int(stats[4])) * bits_b           # LTD/LTP trial reads (a5)
                 + (int(stats[3]) + int(stats[5])) * bits_b)          # conditional writes (a5)
    per_launch_bytes = alg_bytes / max(1, launches)
    per_launch_s = dev_s / max(1, launches) if not dist else (sum(step_ms) / 1e3) / max(1, launches)
    smclk = (clocks.get("sm_max_mhz") or 1965.0)
    peak_smem = SMEM_BYTES_PER_CLK_PER_SM * N_SM * smclk * 1e6 / 1e9   # GB/s, whole chip
    achieved = per_launch_bytes / per_launch_s / 1e9
    roofline = {"bound": "smem", "achieved": achieved, "peak": peak_smem, "unit": "GB/s", "frac": achieved / peak_smem,
                "traffic": None,
                "peak_source": f"derived: 128 B/clk/SM (B300_MICROARCH smem crossbar) x {N_SM} SMs x {smclk:.0f} MHz",
                "alg_bytes_per_launch": per_launch_bytes,
                "note": "latency-bound step loop; see latency_roofline"}

    line = {
        "metric": METRIC, "value": value, "unit": "images/s", "n_gpus": ws, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": 1e3 * dev_s / args.steps, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f32/u2", "data": "synthetic",
        "config": {"workload": WORKLOAD, "n_in": N_IN, "n_exc": N_EXC, "bits": BITS, "T": T_STEPS,
                   "images_per_step": B, "parallelism": f"replicas x{ws}" if ws > 1 else "1 network / 1 GPU",
                   "cluster_size": info["cluster_size"], "threads_per_cta": info["threads"],
                   "smem_bytes_per_cta": info["smem_bytes"],
                   "l2": "flushed between timed steps (256 MiB write)", "membrane": "fp32" if args.membrane == 0 else "Q15.16"},
        "secondary": {"synaptic_events_per_s": ev_rate, "steps_per_s": images * T_STEPS / dev_s,
                      "post_spikes_per_image": int(stats[1]) / (B * args.steps),
                      "act_per_step": int(stats[0]) / (B * args.steps * T_STEPS),
                      "ltd_trials_per_image": int(stats[2]) / (B * args.steps),
                      "ltp_trials_per_image": int(stats[4]) / (B * args.steps),
                      "step_ms_min": min(step_ms), "step_ms_max": max(step_ms),
                      "epochs_per_image": int(stats[8]) / (B * args.steps),
                      "log_stops_per_image": int(stats[9]) / (B * args.steps),
                      "resims_per_image": int(stats[10]) / (B * args.steps),
                      "speculated_column_steps_ratio": int(stats[11]) / max(1, N_EXC * T_STEPS * B * args.steps)},
        "gpu_launches": launches,
        "clocks": clocks,
        "e2e": e2e,
        "roofline": roofline,
        "latency_roofline": floor,
    }
    if rank == 0 and ws == 1 and args.cpu_images > 0:
        line["cpu_baseline"] = cpu_baseline(args.cpu_images)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if dist:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
