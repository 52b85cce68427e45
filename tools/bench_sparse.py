#!/usr/bin/env python
"""NEXT-4 measurement: the Fig. 4 workload (10^3 LIF neurons, 10^4 synapses, no
learning), recurrent, 5-78 Hz rate-coded drive, T = 1000 steps (1 s at dt = 1 ms) per trial, a batch of
independent trials resident in HBM, CUDA events on the launching stream.  Prints one JSON line."""
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
    ap.add_argument("--trials", type=int, default=2048)
    ap.add_argument("--T", type=int, default=1000)
    ap.add_argument("--n-lif", type=int, default=1000)
    ap.add_argument("--n-syn", type=int, default=10000)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--v-spike", type=float, default=64.0)
    a = ap.parse_args()
    import torch
    import paper_conf_date_shelm19_b200 as P
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    net = P.Network(784, 64, 8, P.preset("8b", v_spike=a.v_spike, f_min_hz=5.0, f_max_hz=78.0))
    net.set_stream(stream.cuda_stream)
    off, tgt, q = synthdata.sparse_graph(784, a.n_lif, a.n_syn, bits=8)
    deg = np.diff(off)
    imgs = torch.from_numpy(synthdata.images(a.trials, "fashion", start=50000)).cuda()
    seeds = torch.from_numpy(synthdata.seeds(a.trials, base_seed=11).view(np.int64)).cuda()
    counts = torch.zeros((a.trials, a.n_lif), dtype=torch.int32, device="cuda")
    g = [torch.from_numpy(x).cuda() for x in (off, tgt.view(np.int16), q)]
    net.sparse_run(a.n_lif, g[0], g[1], g[2], imgs, a.T, seeds, counts, None, P.SNN_ASYNC)
    torch.cuda.synchronize()
    st0 = net.sparse_stats().copy()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(a.steps)]
    for e0, e1 in ev:
        e0.record(stream)
        net.sparse_run(a.n_lif, g[0], g[1], g[2], imgs, a.T, seeds, counts, None, P.SNN_ASYNC)
        e1.record(stream)
    torch.cuda.synchronize()
    ms = [e0.elapsed_time(e1) for e0, e1 in ev]
    st = net.sparse_stats() - st0
    t = sum(ms) / 1e3
    n = a.trials * a.steps
    # synaptic events: input spikes x mean input out-degree + neuron spikes x mean neuron out-degree
    ev_syn = float(st[0]) * deg[:784].mean() + float(st[1]) * deg[784:].mean()
    print(json.dumps({"metric": "Fig. 4 workload (10^3 LIF, 10^4 synapses): neuron-steps/s", "value": n * a.T * a.n_lif / t,
                      "unit": "neuron-steps/s", "trials_per_s": n / t, "ms_per_call": sum(ms) / len(ms),
                      "trials_per_call": a.trials, "T": a.T, "synaptic_events_per_s": ev_syn / t,
                      "spikes_per_neuron_per_s_sim": float(st[1]) / (n * a.n_lif * a.T * 1e-3),
                      "n_lif": a.n_lif, "n_syn": a.n_syn}))


if __name__ == "__main__":
    main()
