#!/usr/bin/env python
"""NEXT-1 analysis: the synthetic accuracy proxy and the Fig. 6(b)-style conductance
histogram ("distribution of conductance of all ... synapses") of a network trained with the
P:88 protocol (train, label the neurons with a labelling set, classify an evaluation set), for a grid of
readings of the parameters the paper leaves open (R3 v_spike, R6 t_ref, R7 t_inh).  Every presentation,
inference, labelling and vote runs in the CUDA library (paper_conf_date_shelm19_b200.schedule).

Prints one JSON line per configuration: error rate, distinct winning neurons, labelled neurons, and the
histogram of the learned codes (counts per code value, G = q * 2^-frac_bits).
    python tools/accuracy_proxy.py --grid            # the reading sweep
    python tools/accuracy_proxy.py --table2          # Table II rules x roundings at the chosen reading
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synthdata  # noqa: E402


def run(bits, preset, overrides, n_train, n_label, n_eval, n_exc=400, T=350, kind="mnist"):
    import paper_conf_date_shelm19_b200 as P
    from paper_conf_date_shelm19_b200.schedule import Phase, run_schedule
    tr = synthdata.images(n_train, kind, start=0)
    trs = synthdata.seeds(n_train, base_seed=1)
    li, lc, ls = synthdata.images(n_label, kind, start=50000), synthdata.labels(n_label, 50000), synthdata.seeds(n_label, 2)
    ei, ec, es = synthdata.images(n_eval, kind, start=60000), synthdata.labels(n_eval, 60000), synthdata.seeds(n_eval, 3)
    curve, net = run_schedule(784, n_exc, bits, [Phase(preset, T, n_train, dict(overrides))], tr, trs, li, lc, ls,
                              ei, ec, es, eval_every=n_train)
    w = net.weights()
    q_max = (1 << bits) - 1
    hist = np.bincount(w.reshape(-1).astype(np.int64), minlength=q_max + 1)
    counts = net.infer(ei, T, es)
    labels = net.label(net.infer(li, T, ls), np.ascontiguousarray(lc.astype(np.int32)), 10)
    winners = int((counts.sum(axis=0) > 0).sum())
    return {"error": curve[-1].error, "neurons_spiking_on_eval": winners,
            "labelled_neurons": int((labels >= 0).sum()), "code_hist": hist.tolist() if bits <= 8 else None,
            "mean_G": float(w.mean()) / (1 << bits)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--grid", action="store_true")
    ap.add_argument("--table2", action="store_true")
    ap.add_argument("--train", type=int, default=1000)
    ap.add_argument("--label", type=int, default=500)
    ap.add_argument("--eval", type=int, default=500)
    ap.add_argument("--t-ref", type=int, default=None)
    ap.add_argument("--t-inh", type=int, default=None)
    ap.add_argument("--v-spike", type=float, default=None)
    a = ap.parse_args()
    import torch
    torch.cuda.set_device(0)
    base = {}
    if a.t_ref is not None:
        base["t_ref_steps"] = a.t_ref
    if a.t_inh is not None:
        base["t_inh_steps"] = a.t_inh
    if a.v_spike is not None:
        base["v_spike"] = a.v_spike
    if a.grid:
        for t_ref, t_inh in ((5, 10), (10, 10), (20, 10), (20, 20), (40, 20)):
            for v_spike in (1.0, 2.0, 4.0):
                ov = dict(t_ref_steps=t_ref, t_inh_steps=t_inh, v_spike=v_spike)
                r = run(8, "8b", ov, a.train, a.label, a.eval)
                print(json.dumps({"bits": 8, "rule": "stochastic", **ov, **{k: r[k] for k in
                      ("error", "neurons_spiking_on_eval", "labelled_neurons", "mean_G")}}), flush=True)
    if a.table2:
        for bits, pre in ((2, "2b"), (4, "4b"), (8, "8b")):
            for rule, rnd in (("stochastic", 1), ("deterministic", 0), ("deterministic", 1), ("deterministic", 2)):
                ov = dict(base, stdp_mode=0 if rule == "stochastic" else 1, rounding=rnd)
                r = run(bits, pre, ov, a.train, a.label, a.eval)
                print(json.dumps({"bits": bits, "rule": rule, "rounding": ["trunc", "nearest", "stochastic"][rnd],
                                  **base, **r}), flush=True)


if __name__ == "__main__":
    main()
