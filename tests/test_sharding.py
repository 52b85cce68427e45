"""Column sharding of one network across ranks: a CPU test double of the exchange
protocol, run as world_size-2 `gloo` process groups, must reproduce the unsharded oracle bit for
bit.  Rank r owns a contiguous slice of post-synaptic columns (codes, v, countdown, last_post); the
encoder and last_pre are replicated (every rank draws the same Philox inputs, R13); per step the
ranks exchange one candidate key (HARD) or a candidate count (LAYER) with all_gather, then apply
inhibition locally; LTD/LTP draws are keyed by GLOBAL indices, so the slicing cannot change them.
This pins the host-side protocol the sharded CUDA path (and bench.py's multi-rank mode) relies on.
Q15.16 membranes keep the double exact in Python integers."""
import math
import os

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import oracle as O

N_IN, N_EXC, BITS, T = 64, 20, 8, 60


def _llround(x):
    r = math.floor(abs(x) + 0.5)
    return int(r) if x >= 0 else -int(r)


def _thr(P):
    return math.floor(math.ldexp(P, 32))


def _draw(seed, c0, c1, c2, tag, lane):
    return O.philox4x32_10([c0 & 0xFFFFFFFF, c1, c2, tag], [seed & 0xFFFFFFFF, seed >> 32])[lane]


def shard_worker(rank, world, port, p, q0, image, seed, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    lo, hi = rank * N_EXC // world, (rank + 1) * N_EXC // world
    cols = list(range(lo, hi))
    qmax = 2 ** BITS - 1
    lsb = 2.0 ** -BITS
    dt = p["dt_ms"]
    A = _llround(dt * p["a"] * 65536.0)
    B = _llround(dt * p["b"] * 4294967296.0)
    C = _llround(dt * p["c"] * p["v_spike"] * lsb * 4294967296.0)
    E = _llround(dt * p["c"] * p["i_ext"] * 65536.0)
    Vth, Vreset, Vinit = (_llround(p[k] * 65536.0) for k in ("v_th", "v_reset", "v_init"))
    thr_enc = [_thr((p["f_min_hz"] + (p["f_max_hz"] - p["f_min_hz"]) * x / 255.0) * dt * 1e-3) for x in range(256)]

    def lut(g, tau):
        out = []
        for D in range(4096):
            v = _thr(g * math.exp(-(D * dt) / tau))
            if v == 0:
                break
            out.append(v)
        return out

    pot, dep = lut(p["gamma_pot"], p["tau_pot"]), lut(p["gamma_dep"], p["tau_dep"])
    q = q0[:, lo:hi].astype(np.int64).copy()               # this rank's columns
    v = [Vinit] * len(cols)
    cnt = [0] * len(cols)
    lpost = [-1] * len(cols)
    lpre = [-1] * N_IN                                      # replicated
    raster = np.zeros((T, N_EXC), bool)
    for t in range(T):
        s = [_draw(seed, t, i >> 2, 0, 1, i & 3) < thr_enc[image[i]] for i in range(N_IN)]   # replicated encoder
        for i in range(N_IN):
            if s[i]:
                lpre[i] = t
        cand = [False] * len(cols)
        for k in range(len(cols)):
            S = int(sum(q[i, k] for i in range(N_IN) if s[i]))
            if cnt[k] > 0:
                cnt[k] -= 1
                continue
            x = v[k]
            v[k] = x + A + ((B * x + (1 << 31)) >> 32) + ((C * S + (1 << 15)) >> 16) + E
            cand[k] = v[k] > Vth
        if p["wta_mode"] == 0:
            # local best key (ord(v) << 32 | ~j), exchanged with all_gather -> global winner
            best = 0
            for k in range(len(cols)):
                if cand[k]:
                    key = ((v[k] + (1 << 31)) << 32) | (0xFFFFFFFF - cols[k])
                    best = max(best, key)
            keys = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
            dist.all_gather(keys, torch.tensor([best - (1 << 63)], dtype=torch.int64))
            K = max(int(x.item()) + (1 << 63) for x in keys)
            W = (0xFFFFFFFF - (K & 0xFFFFFFFF)) if K else -1
            spikers = [W] if W >= 0 else []
            total = len(spikers)
        else:
            counts = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
            dist.all_gather(counts, torch.tensor([sum(cand)], dtype=torch.int64))
            total = sum(int(x.item()) for x in counts)
            spikers = [cols[k] for k in range(len(cols)) if cand[k]]
        for k, j in enumerate(cols):
            me = j in spikers
            if me:
                v[k] = Vreset
                cnt[k] = p["t_ref_steps"]
                raster[t, j] = True
            if total and (total >= 2 or not me) and not (p["wta_mode"] == 0 and me):
                cnt[k] = max(cnt[k], p["t_inh_steps"])
                if p["inh_mode"] == 0:
                    v[k] = Vreset
        # LTD on own columns (global j in the draw), then LTP on own spikers
        for i in range(N_IN):
            if not s[i]:
                continue
            for k, j in enumerate(cols):
                if lpost[k] < 0:
                    continue
                D = t - lpost[k]
                if D < len(dep) and _draw(seed, t, i, j >> 2, 2, j & 3) < dep[D]:
                    q[i, k] = max(q[i, k] - 1, 0)
        for k, j in enumerate(cols):
            if j not in spikers:
                continue
            for i in range(N_IN):
                if lpre[i] < 0:
                    continue
                D = t - lpre[i]
                if D < len(pot) and _draw(seed, t, j, i >> 2, 3, i & 3) < pot[D]:
                    q[i, k] = min(q[i, k] + 1, qmax)
            lpost[k] = t
    np.save(os.path.join(out_dir, f"q{rank}.npy"), q)
    np.save(os.path.join(out_dir, f"r{rank}.npy"), raster[:, lo:hi])
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("wta", [0, 1])
def test_column_sharded_protocol_matches_oracle(tmp_path, wta):
    p = O.params("8b", membrane_mode=1, wta_mode=wta, f_min_hz=40.0, f_max_hz=400.0, v_spike=24.0,
                 t_ref_steps=2, t_inh_steps=4, init_seed=21)
    net = O.OracleNet(N_IN, N_EXC, BITS, p)
    q0 = net.weights()
    image = (np.arange(N_IN) * 37 % 256).astype(np.uint8)
    seed = 4242
    net.present(image, T, seed)
    world = 2
    port = 29500 + (os.getpid() % 1000) + 7 * wta
    mp.spawn(shard_worker, args=(world, port, p, q0, image, seed, str(tmp_path)), nprocs=world, join=True)
    q = np.concatenate([np.load(tmp_path / f"q{r}.npy") for r in range(world)], axis=1)
    r = np.concatenate([np.load(tmp_path / f"r{r}.npy") for r in range(world)], axis=1)
    assert r.any(), "the configuration must spike"
    assert np.array_equal(r, O.unpack_bits(net.spikes(), N_EXC))
    assert np.array_equal(q.astype(np.uint8), net.weights())
