"""NEXT-3: the frequency-control schedule as a training driver.

P:87 §III-A: "Frequency control module works in two phases: frequency boost and learning time
reduction."  P:94 §IV-C: the baseline learns at 1-22 Hz with 500 ms per image; with "higher tau_pot
and lower tau_dep" (Table I "high frequency" row) the input range "can be expanded up to 5-78 Hz"
and "learning time for each image is reduced to 100 ms"; Fig. 8(c) plots the moving error rate against
simulation time.

A schedule is a list of phases; each phase presents `n_images` training images for `T` steps with its
own parameter block (Table I row + overrides: the frequency boost changes f_min/f_max and the STDP time
constants, the learning-time reduction changes T).  The conductance codes carry over from phase to phase
(the network is re-created with the next phase's parameters and the codes are copied over).
Every `eval_every` training images the driver freezes the weights and measures the error rate with the
P:88 protocol (NEXT-1): label the neurons with a labelling set, classify an evaluation set.

Host orchestration only: every presentation, inference, labelling and vote runs in the CUDA library.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Callable, List, Optional

import numpy as np

from .snn import SNN_ASYNC, Network, preset


@dataclass
class Phase:
    preset: str                 # Table I row: "2b", "4b", "8b", "hf"
    T: int                      # steps per training image (t_learn in ms at dt = 1 ms)
    n_images: int               # training images presented in this phase
    overrides: dict = field(default_factory=dict)


# baseline 1-22 Hz, 500 ms per image; frequency boost (Table I "high frequency" row, 5-78 Hz) followed
# by learning-time reduction to 100 ms.
def paper_phases(n_baseline: int, n_boost: int, n_reduced: int, bits_preset: str = "8b") -> List[Phase]:
    hf = {k: getattr(preset("hf"), k) for k in ("f_min_hz", "f_max_hz", "gamma_pot", "tau_pot", "gamma_dep",
                                                "tau_dep")}
    return [Phase(bits_preset, 500, n_baseline),
            Phase(bits_preset, 500, n_boost, dict(hf)),
            Phase(bits_preset, 100, n_reduced, dict(hf))]


@dataclass
class CurvePoint:
    images: int                 # training images presented so far
    sim_ms: float               # simulated learning time so far (sum of T * dt)
    device_s: float             # device time spent in training presentations so far
    error: float                # error rate on the evaluation set (unclassified counts as an error)
    phase: int


def run_schedule(n_in: int, n_exc: int, bits: int, phases: List[Phase], train_images, train_seeds,
                 label_images, label_classes, label_seeds, eval_images, eval_classes, eval_seeds,
                 eval_every: int, eval_T: Optional[int] = None, n_classes: int = 10,
                 common: Optional[dict] = None, stream=None,  # stream: a torch.cuda.Stream
                 on_point: Optional[Callable[[CurvePoint], None]] = None):
    """Run the schedule; returns (curve, final Network).  Arrays are numpy (host) or torch CUDA tensors;
    the training images are consumed in order across phases.  eval_T: steps per labelling/evaluation
    image (default: the current phase's T)."""
    import torch
    common = dict(common or {})
    # a dedicated (non-default) stream: the networks launch on it and the timing events are recorded on it
    # (cuda_stream 0 would mean "the handle's own stream" to snn_set_stream)
    tstream = stream if stream is not None else torch.cuda.Stream()
    curve: List[CurvePoint] = []
    net: Optional[Network] = None
    seen, sim_ms, dev_s = 0, 0.0, 0.0
    lab_cls = np.ascontiguousarray(np.asarray(label_classes, dtype=np.int32))
    ev_cls = np.asarray(eval_classes, dtype=np.int64)

    def evaluate(phase_idx: int, T_eval: int):
        cl = net.infer(label_images, T_eval, label_seeds)
        labels = net.label(cl, lab_cls, n_classes)
        ce = net.infer(eval_images, T_eval, eval_seeds)
        pred = net.classify(ce, labels, n_classes)
        pt = CurvePoint(seen, sim_ms, dev_s, float(np.mean(pred != ev_cls)), phase_idx)
        curve.append(pt)
        if on_point:
            on_point(pt)

    for pi, ph in enumerate(phases):
        params = preset(ph.preset, **{**common, **ph.overrides})
        new = Network(n_in, n_exc, bits, params)
        new.set_stream(tstream.cuda_stream)
        if net is not None:
            new.set_weights(net.weights())          # the learned codes carry over (P:87 two-phase module)
            net.close()
        net = new
        done = 0
        while done < ph.n_images:
            nb = min(eval_every - (seen % eval_every), ph.n_images - done)
            sl = slice(seen, seen + nb)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(tstream)
            net.present_batch(train_images[sl], ph.T, train_seeds[sl], None, flags=SNN_ASYNC)
            e1.record(tstream)
            torch.cuda.synchronize()
            dev_s += e0.elapsed_time(e1) / 1e3
            seen += nb
            done += nb
            sim_ms += nb * ph.T * params.dt_ms
            if seen % eval_every == 0:
                evaluate(pi, eval_T or ph.T)
    if not curve or curve[-1].images != seen:
        evaluate(len(phases) - 1, eval_T or phases[-1].T)
    return curve, net
