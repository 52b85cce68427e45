#!/usr/bin/env python
"""NEXT-3 measurement: the paper's two-phase frequency-control schedule against
the baseline schedule on synthetic MNIST-shaped data.  Prints one JSON line per schedule with the error
curve (P:88 labelling + inference protocol every --eval-every images) over simulated and device time."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synthdata  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n-exc", type=int, default=400)
    ap.add_argument("--bits", type=int, default=8)
    ap.add_argument("--train", type=int, default=3000)
    ap.add_argument("--eval-every", type=int, default=250)
    ap.add_argument("--n-label", type=int, default=1000)
    ap.add_argument("--n-eval", type=int, default=2000)
    ap.add_argument("--t-ref", type=int, default=None, help="reading R6b: e.g. --t-ref 10 --t-inh 10")
    ap.add_argument("--t-inh", type=int, default=None)
    a = ap.parse_args()
    common = {}
    if a.t_ref is not None:
        common["t_ref_steps"] = a.t_ref
    if a.t_inh is not None:
        common["t_inh_steps"] = a.t_inh
    import torch
    from paper_conf_date_shelm19_b200 import schedule as S
    torch.cuda.set_device(0)
    pre = {2: "2b", 4: "4b", 8: "8b"}[a.bits]
    tr = synthdata.images(a.train, "mnist")
    trs = synthdata.seeds(a.train, base_seed=41)
    li = synthdata.images(a.n_label, "mnist", start=100000)
    lc = synthdata.labels(a.n_label, start=100000)
    ls = synthdata.seeds(a.n_label, base_seed=42)
    ei = synthdata.images(a.n_eval, "mnist", start=200000)
    ec = synthdata.labels(a.n_eval, start=200000)
    es = synthdata.seeds(a.n_eval, base_seed=43)
    third = a.train // 3
    schedules = {
        "baseline (1-22 Hz, 500 ms)": [S.Phase(pre, 500, a.train)],
        "two-phase (boost to 5-78 Hz, then 100 ms)": S.paper_phases(third, third, a.train - 2 * third, pre),
        "high frequency from the start (5-78 Hz, 100 ms)": [S.paper_phases(0, 0, a.train, pre)[2]],
    }
    for name, phases in schedules.items():
        curve, net = S.run_schedule(784, a.n_exc, a.bits, phases, tr, trs, li, lc, ls, ei, ec, es,
                                    eval_every=a.eval_every, eval_T=350, common=common)
        pts = [dict(images=p.images, sim_s=p.sim_ms / 1e3, device_s=p.device_s, error=p.error, phase=p.phase)
               for p in curve]
        print(json.dumps({"schedule": name, "n_exc": a.n_exc, "bits": a.bits, "train_images": a.train, **common,
                          "train_images_per_s": a.train / curve[-1].device_s, "final_error": curve[-1].error,
                          "curve": pts}), flush=True)
        net.close()


if __name__ == "__main__":
    main()
