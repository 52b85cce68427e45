#!/usr/bin/env python
"""Benchmark of the simulate-and-learn path (driver contract).

Workload (BASELINE.json metric "synaptic events/sec & training images/sec (784->6400, 2-bit)"):
config C4 -- one 784 -> 6400 LIF network, 2-bit codes, stochastic STDP (Table I "2 bit" row),
fashion-shaped synthetic images, T = 350 steps (350 ms at dt = 1 ms), 1-22 Hz, HARD WTA, fp32
membranes.  A "step" = one snn_present_batch launch presenting B images back to back (online
learning: the images of a step are sequential by construction).  value = training images/s with
inputs resident in HBM; secondary = synaptic events/s (sum_t act(t) * n_exc).

Multi-GPU (torchrun, N > 1), --mode:
  replicas (default): one independent network per GPU, no data-path collective ("scaling": "weak");
  shard: ONE network whose 6400 columns are split over the N GPUs (include/snn.h snn_create_shard):
         per post-spike epoch the shards exchange 16-byte summaries through CUDA-IPC mailboxes over
         NVLink ("scaling": "strong": every rank presents the same images);
  shard-weak: one network of 6400*N columns, 6400 per GPU, same exchange ("scaling": "weak");
  ensemble: C5, --nets independent 784->400 networks per GPU (bits (2,4,8)[k%3]) presented with one
         snn_present_many per step, replicas across GPUs (its own metric line).
--local-shards K (N = 1): the one network split into K shards on this GPU, presented in one launch
(K clusters exchanging through L2 mailboxes) -- more SMs per network.

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


def cpu_info() -> dict:
    """CPU model and core counts of the host the oracle runs on (lscpu, else /proc/cpuinfo)."""
    info = {"model": None, "logical_cpus": os.cpu_count(), "usable_cpus": len(os.sched_getaffinity(0))}
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            k, _, v = line.partition(":")
            if k.strip() == "Model name":
                info["model"] = v.strip()
            elif k.strip() in ("Socket(s)", "Core(s) per socket", "Thread(s) per core"):
                info[k.strip().lower().replace("(s)", "s").replace(" ", "_")] = v.strip()
    except Exception:
        pass
    if info["model"] is None:
        try:
            for line in open("/proc/cpuinfo"):
                if line.startswith("model name"):
                    info["model"] = line.split(":", 1)[1].strip()
                    break
        except OSError:
            pass
    return info


def _oracle_images(mode: int, n_images: int) -> float:
    """Seconds for the oracle to present n_images C4 images (784->6400, 2-bit, T=350) in membrane mode `mode`."""
    from oracle import oracle as O
    p = O.params("2b", membrane_mode=mode, init_seed=1)
    net = O.OracleNet(N_IN, N_EXC, BITS, p)
    imgs = synthdata.images(n_images, "fashion", start=1000)
    seeds = synthdata.seeds(n_images, base_seed=3)
    t0 = time.perf_counter()
    for k in range(n_images):
        net.present(imgs[k], T_STEPS, int(seeds[k]))
    return time.perf_counter() - t0


def _c5_pinned(args):
    k, cpu = args
    os.sched_setaffinity(0, {cpu})
    return _c5_worker_unpinned(k)


def _c5_worker_unpinned(k: int) -> float:
    """One C5 network (784->400, bits {2,4,8}[k % 3], its Table I row, seed k) presenting 2 MNIST-shaped
    images; returns the seconds it took."""
    from oracle import oracle as O
    bits = (2, 4, 8)[k % 3]
    net = O.OracleNet(N_IN, 400, bits, O.params({2: "2b", 4: "4b", 8: "8b"}[bits], init_seed=1 + k))
    imgs = synthdata.images(2, "mnist", start=10 * k)
    seeds = synthdata.seeds(2, base_seed=100 + k)
    t0 = time.perf_counter()
    for x, sd in zip(imgs, seeds):
        net.present(x, T_STEPS, int(sd))
    return time.perf_counter() - t0


def cpu_baseline(n_images: int) -> dict:
    """The oracle as it stands (never tuned), on the host: C4 on ONE pinned core in both membrane modes (the
    line's value is the fp32 mode, the bench's), plus the all-cores C5 ensemble figure: one
    784->400 network per core, min(64, cores) networks in parallel."""
    cpus = sorted(os.sched_getaffinity(0))
    old = set(cpus)
    os.sched_setaffinity(0, {cpus[0]})                  # taskset -c <first usable core>
    try:
        t_fp32 = _oracle_images(0, n_images)
        t_fixed = _oracle_images(1, n_images)
    finally:
        os.sched_setaffinity(0, old)
    out = {"value": n_images / t_fp32, "unit": "images/s", "cores": 1, "kind": "oracle",
           "sample": f"{n_images} fashion images of C4 (784->6400, 2-bit, T=350) via oracle_present, fp32 membranes, "
                     f"pinned to core {cpus[0]}",
           "fixed_q15_16": {"value": n_images / t_fixed, "unit": "images/s", "cores": 1},
           "cpu": cpu_info()}
    try:
        import multiprocessing as mp
        n = min(64, len(cpus))
        ctx = mp.get_context("spawn")
        t0 = time.perf_counter()
        with ctx.Pool(n) as pool:
            secs = pool.map(_c5_pinned, [(k, cpus[k % len(cpus)]) for k in range(n)])
        wall = time.perf_counter() - t0
        out["c5_all_cores"] = {"value": 2 * n / max(secs), "unit": "images/s", "cores": n, "networks": n,
                               "sample": f"{n} C5 networks (784->400, bits (2,4,8)[k%3], Table I rows), one per "
                                         f"pinned core, 2 MNIST-shaped images each, T=350; value = images / slowest "
                                         f"network's time", "wall_s_incl_spawn": wall}
    except Exception as e:                              # noqa: BLE001 -- a missing pool must not sink the bench
        out["c5_all_cores"] = {"unavailable": str(e)[:200]}
    return out


def run_ensemble(args):
    """C5: an ensemble of independent 784 -> 400 networks, --nets per GPU (bit widths (2,4,8)[k%3],
    each with its Table I row, seed = global network index), MNIST-shaped images, T = 350.  Every rank presents
    its own group with one snn_present_many per step (one launch per bit width); replicas across ranks with no
    data-path collective ("scaling": "weak").  Device time (CUDA events on the launching stream), max over
    ranks; value = images of all networks of all ranks / that time."""
    import torch
    import paper_conf_date_shelm19_b200 as P
    ws, rank, local = _dist_env()
    dev = torch.device("cuda", local % max(1, torch.cuda.device_count()))
    torch.cuda.set_device(dev)
    dist = None
    if ws > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl" if torch.cuda.device_count() >= ws else "gloo",
                                **({"device_id": dev} if torch.cuda.device_count() >= ws else {}))
    stream = torch.cuda.Stream(dev)
    torch.cuda.set_stream(stream)
    B, NE = args.images_per_step, 400
    nets, imgs, seeds = [], [], []
    for k in range(args.nets):
        g = rank * args.nets + k
        bits = (2, 4, 8)[g % 3]
        n = P.Network(N_IN, NE, bits, P.preset({2: "2b", 4: "4b", 8: "8b"}[bits], init_seed=1 + g, cluster_size=2))
        n.set_stream(stream.cuda_stream)
        nets.append(n)
        tot = B * (args.warmup + args.steps)
        imgs.append(torch.from_numpy(synthdata.images(tot, "mnist", start=10000 * g)).to(dev))
        seeds.append(torch.from_numpy(synthdata.seeds(tot, base_seed=200 + g).view(np.int64)).to(dev))
    flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=dev)
    sl = lambda s: slice(s * B, (s + 1) * B)  # noqa: E731
    for s in range(args.warmup):
        P.present_many(nets, [x[sl(s)] for x in imgs], T_STEPS, [x[sl(s)] for x in seeds])
    torch.cuda.synchronize()
    for n in nets:
        n.reset_stats()
    sampler = ClockSampler(local)
    sampler.start()
    time.sleep(0.15)
    if dist:
        dist.barrier()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    for i in range(args.steps):
        flush.fill_(i & 0xFF)
        s = args.warmup + i
        ev[i][0].record(stream)
        P.present_many(nets, [x[sl(s)] for x in imgs], T_STEPS, [x[sl(s)] for x in seeds])
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    if dist:
        dist.barrier()
    clocks = sampler.stop()
    dev_s = sum(a.elapsed_time(b) for a, b in ev) / 1e3
    images = args.nets * B * args.steps
    events = sum(int(n.stats()[0]) for n in nets) * NE
    if dist:
        t = torch.tensor([dev_s], dtype=torch.float64, device=dev if torch.cuda.device_count() >= ws else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dev_s = float(t.item())
        tot = torch.tensor([images, events], dtype=torch.float64, device=t.device)
        dist.all_reduce(tot, op=dist.ReduceOp.SUM)
        images, events = int(tot[0].item()), int(tot[1].item())
    if rank == 0:
        print(json.dumps({
            "metric": "C5 ensemble training images/s (784->400, bits {2,4,8})", "value": images / dev_s,
            "unit": "images/s", "n_gpus": ws, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * dev_s / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f32/u2-u8", "data": "synthetic",
            "config": {"workload": "C5: independent 784->400 networks, bits (2,4,8)[k%3], Table I rows, MNIST-shaped, "
                                   "T=350", "nets_per_gpu": args.nets, "images_per_net_per_step": B,
                       "parallelism": f"{args.nets} networks per GPU x {ws} GPU(s), replicas",
                       "l2": "flushed between timed steps (256 MiB write)"},
            "secondary": {"synaptic_events_per_s": events / dev_s, "per_net_images_per_s": images / dev_s /
                          (args.nets * ws)},
            "clocks": clocks}), flush=True)
    if dist:
        dist.barrier()
        dist.destroy_process_group()


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
    ap.add_argument("--mode", default="replicas", choices=["replicas", "shard", "shard-weak", "ensemble"],
                    help="replicas: one C4 network per GPU; shard: ONE C4 network's 6400 columns split over the GPUs "
                         "(strong); shard-weak: a 6400*N-column network, 6400 columns per GPU (weak); ensemble: C5, "
                         "--nets 784->400 networks per GPU")
    ap.add_argument("--nets", type=int, default=8, help="ensemble mode: networks per GPU")
    ap.add_argument("--local-shards", type=int, default=1, help="shards of the network on this GPU (N = 1)")
    ap.add_argument("--no-infer", action="store_true", help="skip the NEXT-1 inference measurement")
    ap.add_argument("--infer-images", type=int, default=4096, help="images per inference call")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)
    if args.mode == "ensemble":
        return run_ensemble(args)

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
    sharded = ws > 1 and args.mode in ("shard", "shard-weak")
    n_exc_net = N_EXC * ws if (sharded and args.mode == "shard-weak") else N_EXC   # columns of the whole network
    K = args.local_shards if ws == 1 else 1
    net_rank = 0 if sharded else rank           # shards of one network share seeds and images

    def make_runner():
        """-> (present(imgs, seeds, counts, flags), stats(), nets) for the configured layout."""
        params = P.preset("2b", membrane_mode=args.membrane, init_seed=1 + net_rank,
                          cluster_size=args.cluster_size, engine=args.engine)
        if sharded:
            n = P.Network(N_IN, n_exc_net, BITS, params, shard=(rank, ws))
            n.set_stream(stream.cuda_stream)
            hs = [None] * ws
            dist.all_gather_object(hs, n.ipc_handle())
            n.connect(hs)
            nets = [n]
        elif K > 1:
            nets = [P.Network(N_IN, N_EXC, BITS, params, shard=(r, K)) for r in range(K)]
            P.link_shards(nets)
            for n in nets:
                n.set_stream(stream.cuda_stream)
        else:
            nets = [P.Network(N_IN, N_EXC, BITS, params)]
            nets[0].set_stream(stream.cuda_stream)
        if K > 1:
            def present(imgs, seeds, counts, flags=0):
                P.present_many(nets, [imgs] * K, T_STEPS, [seeds] * K)
        else:
            def present(imgs, seeds, counts, flags=0):
                nets[0].present_batch(imgs, T_STEPS, seeds, counts, flags=flags)
        return present, nets

    present, nets = make_runner()
    net = nets[0]
    info = net.info()

    n_steps_total = args.warmup + args.steps
    pool_n = B * n_steps_total
    imgs_h = synthdata.images(pool_n, "fashion", start=net_rank * 100000)
    seeds_h = synthdata.seeds(pool_n, base_seed=1 + net_rank)
    imgs_d = torch.from_numpy(imgs_h).to(dev)
    seeds_d = torch.from_numpy(seeds_h.view(np.int64)).to(dev)
    counts_d = torch.zeros(pool_n, dtype=torch.int32, device=dev)
    flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=dev)   # > 126 MB L2

    def step(k, flags=0):
        sl = slice(k * B, (k + 1) * B)
        present(imgs_d[sl], seeds_d[sl], counts_d[sl], flags | P.SNN_ASYNC)

    for k in range(args.warmup):
        step(k)
    torch.cuda.synchronize()
    for n in nets:
        n.reset_stats()
    launches0 = sum(n.info()["launches"] for n in nets)
    profiled = K == 1                                 # single-handle presentations record kernel events
    if profiled:
        net0 = nets[0]
        net0.set_profile(True)

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
    kern_ms, kern_n = nets[0].profile() if profiled else (None, 0)
    if profiled:
        nets[0].set_profile(False)
    dev_s = sum(step_ms) / 1e3
    stats = net.stats()
    for n in nets[1:]:                 # per-shard trial / event counters add up; [0], [1], [6..8] are network-wide
        stats[2:6] += n.stats()[2:6]
    launches = sum(n.info()["launches"] for n in nets) - launches0
    images = B * args.steps
    events = int(stats[0]) * n_exc_net                 # every column of the network (all shards)
    # max over ranks of the device time
    if dist:
        t = torch.tensor([dev_s], device=coll_dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dev_s = float(t.item())
        if not sharded:                # replicas: every rank trained its own network on its own images
            tot = torch.tensor([images, events], device=coll_dev, dtype=torch.float64)
            dist.all_reduce(tot, op=dist.ReduceOp.SUM)
            images, events = int(tot[0].item()), int(tot[1].item())
    value = images / dev_s
    ev_rate = events / dev_s

    # ---- latency floor: the same launch shape (B images, same cluster) doing only the
    # synchronisation skeleton of the path -- per epoch (lean kernel: the handle's measured epochs per image) --
    # timed live with CUDA events around the kernel on its stream; frac = t_floor / t_kernel per image
    floor = None
    if not args.no_floor and args.engine == 0 and info.get("lean") and profiled and kern_n:
        net.set_profile(True)
        for i in range(3):
            step(args.warmup + i, flags=P.snn.SNN_FLOOR_PROBE)
        fl_ms, fl_n = net.profile()
        net.set_profile(False)
        t_img = 1e3 * (kern_ms / kern_n) / B
        t_fl = 1e3 * (fl_ms / fl_n) / B
        floor = {"kind": "lean kernel, same launch shape: per epoch only the early-stop signal, warp/CTA summaries, "
                         "DSMEM stores, cluster barrier and decision (SNN_FLOOR_PROBE), measured live",
                 "epochs_per_image": int(stats[8]) / (B * args.steps), "t_floor_us_per_image": t_fl,
                 "t_kernel_us_per_image": t_img, "frac": t_fl / t_img}
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
    present2, nets2 = make_runner()
    d2h = B * 4 if K == 1 else 16 * 8

    def step2(sl):
        present2(imgs_pin[sl], seeds_pin[sl], counts_pin[sl])
        if K > 1:                      # synchronous present_many: read the post-spike counter back
            nets2[0].stats()
    for k in range(args.warmup):
        step2(slice(k * B, (k + 1) * B))
    if dist:
        dist.barrier()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for i in range(args.steps):
        k = args.warmup + i
        sl = slice(k * B, (k + 1) * B)
        step2(sl)                      # synchronous: result on host
    torch.cuda.synchronize()
    e2e_s = time.perf_counter() - t0
    if dist:
        t = torch.tensor([e2e_s], device=coll_dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_s = float(t.item())
    e2e = {"value": images / e2e_s, "unit": "images/s", "h2d_bytes_per_step": B * (N_IN + 8) * K,
           "d2h_bytes_per_step": d2h, "timing": "host wall clock around synchronous presentation calls"}

    # ---- roofline of the dominant kernel (present_kernel; one launch per step)
    bits_b = BITS / 8.0
    cols_here = n_exc_net // ws if sharded else N_EXC                  # columns this rank's kernel integrates
    alg_bytes = (int(stats[0]) * cols_here * bits_b                   # integration reads (a2)
                 + (int(stats[2]) + int(stats[4])) * bits_b           # LTD/LTP trial reads (a5)
                 + (int(stats[3]) + int(stats[5])) * bits_b)          # conditional writes (a5)
    # dominant kernel = the presentation kernel (one launch per step); its time comes from the CUDA events the
    # library records around it on the launching stream (snn_set_profile), else the whole step
    n_main = kern_n if (profiled and kern_n) else args.steps
    per_launch_bytes = alg_bytes / max(1, n_main)
    per_launch_s = (kern_ms / 1e3 / kern_n) if (profiled and kern_n) else (sum(step_ms) / 1e3) / args.steps
    smclk = (clocks.get("sm_max_mhz") or 1965.0)
    peak_smem = SMEM_BYTES_PER_CLK_PER_SM * N_SM * smclk * 1e6 / 1e9   # GB/s, whole chip
    achieved = per_launch_bytes / per_launch_s / 1e9
    traffic, traffic_src = None, "no committed ncu --set full capture at this launch shape"
    try:                               # dram bytes of ONE launch of the same shape, from a committed capture
        cap = json.load(open(os.path.join(ROOT, "profiles", "ncu_full_latest.json")))
        if cap.get("images_per_launch") == B and cap.get("n_exc") == N_EXC and K == 1 and not sharded:
            traffic = cap["dram_bytes_per_launch"]
            traffic_src = f"profiles/ncu_full_latest.json ({cap['kernel']}, {cap['source']})"
    except (OSError, ValueError, KeyError):
        pass
    roofline = {"bound": "smem", "achieved": achieved, "peak": peak_smem, "unit": "GB/s", "frac": achieved / peak_smem,
                "traffic": traffic, "traffic_source": traffic_src,
                "peak_source": f"derived: 128 B/clk/SM (B300_MICROARCH smem crossbar) x {N_SM} SMs x {smclk:.0f} MHz",
                "alg_bytes_per_launch": per_launch_bytes,
                "kernel": "present_lean_kernel" if info.get("lean") else "present_event_kernel",
                "kernel_ms_per_launch": 1e3 * per_launch_s,
                "kernel_share_of_step": (kern_ms / sum(step_ms)) if (profiled and kern_n) else None,
                "note": "latency-bound step loop; see latency_roofline"}

    # ---- NEXT-1: inference with the learned weights frozen, images independent.  Device-timed
    # (CUDA events on the launching stream), images resident in HBM.  Dominant kernel: infer_kernel, bound by
    # FP32/INT issue: per column-step the LIF recipe is 7 lane-ops (I2F, FMUL, FADD, 3 FFMA, FSETP), per
    # synaptic event 1 integer add; peak = 148 SMs x 128 lanes x SM clock.
    inference = None
    if K == 1 and not args.no_infer and not sharded:
        # data-parallel over ranks: every rank classifies its own image range with its own network
        nb = args.infer_images
        iimgs = torch.from_numpy(synthdata.images(nb, "fashion", start=200000 + rank * nb)).to(dev)
        iseeds = torch.from_numpy(synthdata.seeds(nb, base_seed=99).view(np.int64)).to(dev)
        icounts = torch.zeros((nb, N_EXC), dtype=torch.int32, device=dev)
        net.infer(iimgs, T_STEPS, iseeds, icounts, flags=P.SNN_ASYNC)
        torch.cuda.synchronize()
        st0 = net.infer_stats().copy()
        iev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(3)]
        for e0, e1 in iev:
            flush.fill_(7)
            e0.record(stream)
            net.infer(iimgs, T_STEPS, iseeds, icounts, flags=P.SNN_ASYNC)
            e1.record(stream)
        torch.cuda.synchronize()
        ims = [a.elapsed_time(b) for a, b in iev]
        ist = (net.infer_stats() - st0).astype(np.float64)
        its = sum(ims) / 1e3
        n_inf = 3 * nb
        if dist:                               # max-over-ranks device time, totals summed over ranks
            t = torch.tensor([its], device=coll_dev, dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            its = float(t.item())
            tot = torch.tensor([float(ist[0]), float(ist[1]), float(ist[2]), float(n_inf)], device=coll_dev,
                               dtype=torch.float64)
            dist.all_reduce(tot, op=dist.ReduceOp.SUM)
            ist = np.array([tot[0].item(), tot[1].item(), tot[2].item()])
            n_inf = int(tot[3].item())
        lane_ops = 7.0 * float(ist[2]) + float(ist[0]) * N_EXC
        smclk_i = (clocks.get("sm_max_mhz") or 1965.0)
        peak_ops = ws * N_SM * 128 * smclk_i * 1e6 / 1e12
        inference = {"metric": "inference images/s (learned weights frozen, P:88 labelling/inference protocol)",
                     "value": n_inf / its, "unit": "images/s", "images_per_call": nb, "ms_per_call": 1e3 * its / 3,
                     "n_gpus": ws, "scaling": "weak",
                     "synaptic_events_per_s": float(ist[0]) * N_EXC / its,
                     "post_spikes_per_image": float(ist[1]) / n_inf,
                     "roofline": {"bound": "alu", "achieved": lane_ops / its / 1e12, "peak": peak_ops,
                                  "unit": "Tlane-op/s", "frac": lane_ops / its / 1e12 / peak_ops,
                                  "work": "7 lane-ops per column-step that ran the LIF recipe (not refractory or "
                                          "inhibited; counted by the kernel) + 1 per synaptic event",
                                  "lif_column_steps_per_image": float(ist[2]) / n_inf,
                                  "peak_source": f"derived: {ws} GPU(s) x 148 SMs x 128 FP32/INT lanes x {smclk_i:.0f} MHz"}}

    line = {
        "metric": METRIC, "value": value, "unit": "images/s", "n_gpus": ws, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": 1e3 * dev_s / args.steps, "higher_is_better": True,
        "scaling": "strong" if (sharded and args.mode == "shard") else "weak", "vs_baseline": None, "dtype": "f32/u2", "data": "synthetic",
        "config": {"workload": WORKLOAD, "n_in": N_IN, "n_exc": n_exc_net, "bits": BITS, "T": T_STEPS,
                   "images_per_step": B,
                   "parallelism": (f"1 network of {n_exc_net} columns, {n_exc_net // ws} per GPU over {ws} GPUs"
                                   if sharded else
                                   f"replicas x{ws}" if ws > 1 else
                                   f"1 network in {K} shards on 1 GPU" if K > 1 else "1 network / 1 GPU"),
                   "cluster_size": info["cluster_size"], "threads_per_cta": info["threads"],
                   "smem_bytes_per_cta": info["smem_lean"] if info.get("lean") else info["smem_bytes"],
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
        "inference": inference,
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
