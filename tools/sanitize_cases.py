#!/usr/bin/env python
"""Small GPU workloads for compute-sanitizer.  Each case runs one kernel
family at a shape small enough for racecheck/synccheck/memcheck to finish in seconds, and checks the
result against the CPU oracle so a sanitizer run is also a parity run.  Usage (on the GPU box):

    compute-sanitizer --tool racecheck --racecheck-report hazard python tools/sanitize_cases.py lean_c1
    python tools/sanitize_cases.py --list
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synthdata  # noqa: E402
from oracle import oracle as O  # noqa: E402


def _net(n_in, n_exc, bits, p, engine=0):
    import paper_conf_date_shelm19_b200 as P
    return P.Network(n_in, n_exc, bits, P.params_from_dict(p, engine=engine)), O.OracleNet(n_in, n_exc, bits, p)


def _batch(g, o, imgs, T, seeds):
    counts = np.zeros(len(imgs), np.int32)
    g.present_batch(imgs, T, seeds, counts)
    for img, sd in zip(imgs, seeds):
        o.present(img, T, int(sd))
    assert np.array_equal(g.weights(), o.weights()), "codes"
    assert np.array_equal(g.spikes(), o.spikes()), "raster"


def learn(n_exc, bits, preset, engine, cs, n_img, T, mode=1, **kw):
    p = O.params(preset, membrane_mode=mode, init_seed=3, cluster_size=cs, **kw)
    g, o = _net(784, n_exc, bits, p, engine)
    _batch(g, o, synthdata.images(n_img, "fashion", start=11), T, synthdata.seeds(n_img, base_seed=5))
    return g.info()


def infer():
    p = O.params("2b", membrane_mode=1, init_seed=3)
    g, o = _net(784, 512, 2, p)
    imgs = synthdata.images(6, "fashion", start=21)
    seeds = synthdata.seeds(6, base_seed=9)
    c = g.infer(imgs, 120, seeds)
    for k in range(6):
        o.present_ex(imgs[k], 120, int(seeds[k]), flags=O.ORACLE_NO_LEARN)
        assert np.array_equal(c[k], O.unpack_bits(o.spikes(), 512).sum(axis=0)), k
    lab = g.label(c, np.arange(6, dtype=np.int32) % 3, 3)
    g.classify(c, lab, 3)


def sparse():
    import paper_conf_date_shelm19_b200 as P
    net = P.Network(784, 64, 8, P.preset("8b", v_spike=64.0, f_min_hz=5.0, f_max_hz=78.0))
    off, tgt, q = synthdata.sparse_graph(784, 200, 2000, bits=8)
    imgs = synthdata.images(4, "fashion", start=7)
    seeds = synthdata.seeds(4, base_seed=3)
    net.sparse_run(200, off, tgt.view(np.int16), q, imgs, 100, seeds)


def shards(world=2):
    import paper_conf_date_shelm19_b200 as P
    p = O.params("2b", membrane_mode=1, init_seed=3)
    sh = [P.Network(784, 512, 2, P.params_from_dict(p), shard=(r, world)) for r in range(world)]
    P.link_shards(sh)
    o = O.OracleNet(784, 512, 2, p)
    imgs = synthdata.images(2, "fashion", start=3)
    seeds = synthdata.seeds(2, base_seed=4)
    P.present_many(sh, [imgs] * world, 150, [seeds] * world)
    for img, sd in zip(imgs, seeds):
        o.present(img, 150, int(sd))
    assert np.array_equal(np.concatenate([s.weights() for s in sh], axis=1), o.weights())


def step_shards(bits, world=2, n_exc=256, preset="16b", **kw):
    """per-step engine column shards (per-step mailbox exchange), 16-bit codes or binary32 conductances"""
    import paper_conf_date_shelm19_b200 as P
    p = O.params(preset, init_seed=3, **kw)
    sh = [P.Network(784, n_exc, bits, P.params_from_dict(p, engine=1), shard=(r, world)) for r in range(world)]
    P.link_shards(sh)
    o = O.OracleNet(784, n_exc, bits, p)
    imgs = synthdata.images(2, "fashion", start=3)
    seeds = synthdata.seeds(2, base_seed=4)
    P.present_many(sh, [imgs] * world, 80, [seeds] * world)
    for img, sd in zip(imgs, seeds):
        o.present(img, 80, int(sd))
    assert np.array_equal(np.concatenate([s.weights() for s in sh], axis=1), o.weights())


CASES = {
    # lean kernel (HARD + RESET + stochastic): C1 shape (one CTA) and a 16-CTA C4-like slice
    "lean_c1": lambda: learn(100, 8, "8b", 0, 0, 3, 100),
    "lean_c4s": lambda: learn(512, 2, "2b", 0, 16, 3, 150),
    "lean_c4s_fp32": lambda: learn(512, 2, "2b", 0, 16, 2, 150, mode=0),
    "lean_c2": lambda: learn(400, 8, "8b", 0, 0, 3, 200),
    # general event kernel (HOLD inhibition forces re-simulation) and LAYER mode
    "general_c1": lambda: learn(100, 8, "8b", 2, 0, 3, 100),
    "general_hold": lambda: learn(400, 8, "8b", 0, 0, 2, 200, inh_mode=1),
    "general_layer_det": lambda: learn(400, 8, "8b", 0, 0, 2, 200, wta_mode=1, stdp_mode=1, rounding=2),
    "general_c4s": lambda: learn(512, 2, "2b", 2, 16, 2, 150),
    # per-step engine (DSMEM exchange every step) and 16-bit codes (step engine only)
    "step_c1": lambda: learn(100, 8, "8b", 1, 0, 2, 100),
    "step_c4s": lambda: learn(512, 2, "2b", 1, 16, 2, 120),
    "step_16b": lambda: learn(200, 16, "16b", 0, 0, 2, 80),
    # LAYER WTA on the lean kernel; binary32 conductances (R28) on the per-step engine; per-step column shards
    "lean_layer": lambda: learn(400, 8, "8b", 0, 0, 2, 200, wta_mode=1),
    "step_fp32": lambda: learn(200, 32, "16b", 0, 0, 2, 80, mode=0),
    "step_fp32_det": lambda: learn(200, 32, "16b", 0, 0, 2, 80, mode=0, stdp_mode=1, wta_mode=1),
    "step_shards_16b": lambda: step_shards(16, rounding=2, membrane_mode=1),
    "step_shards_fp32": lambda: step_shards(32, world=3),
    "infer": infer,
    "sparse": sparse,
    "shards": shards,
}


if __name__ == "__main__":
    if len(sys.argv) < 2 or sys.argv[1] == "--list":
        print(" ".join(CASES))
        sys.exit(0)
    import torch
    torch.cuda.set_device(0)
    for name in sys.argv[1:]:
        out = CASES[name]()
        print(f"case {name} ok {out if out else ''}", flush=True)
