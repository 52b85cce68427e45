"""Column sharding of one network across ranks: CPU test doubles of the exchange
protocols, run as world_size-2 `gloo` process groups, must reproduce the unsharded oracle bit for
bit.  The first double exchanges once per STEP (SURVEY §8(e)'s all_gather reading, every mode): the protocol
the per-step engine's shards ship (best key for HARD, summed count for LAYER); the second,
test_per_epoch_summary_protocol_matches_oracle, is the event engines' protocol: one 16-byte summary per
post-spike EPOCH.  Rank r owns a contiguous slice of post-synaptic columns (codes, v, countdown, last_post); the
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


# ---------------------------------------------------------------------------------------------------------
# The protocol the product ships: not one exchange per step but one per post-spike EPOCH.
# Every rank runs its own columns ahead from the epoch start k0 until their first crossing (integration,
# LIF and the in-order eq.(7) LTD of its columns, R14), publishes a 16-byte summary (earliest crossing step,
# best WTA key at that step), and every rank applies the same reduction to the gathered summaries: t* = the
# earliest step, W = the largest key at t*.  Each rank then commits [k0, t*] (RESET inhibition, R7: every
# column other than W is reset and held, W gets t_ref; LTD with the old last_post, then LTP of W on W's rank,
# then last_post) and the next epoch starts at t* + 1.  HARD + RESET + stochastic STDP (the lean kernel's mode).
def epoch_worker(rank, world, port, p, q0, image, seed, out_dir):
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
    # the encoder is replicated: every rank draws the whole input raster from the same counters (R13)
    S_in = [[_draw(seed, t, i >> 2, 0, 1, i & 3) < thr_enc[image[i]] for i in range(N_IN)] for t in range(T)]

    def lif(x, S):
        return x + A + ((B * x + (1 << 31)) >> 32) + ((C * S + (1 << 15)) >> 16) + E

    def ltd(q, lpost, t):                       # eq.(7) at the pre spikes of step t, old last_post (R10, R14)
        for i in range(N_IN):
            if S_in[t][i]:
                for k, j in enumerate(cols):
                    if lpost[k] >= 0 and t - lpost[k] < len(dep) and _draw(seed, t, i, j >> 2, 2, j & 3) < dep[t - lpost[k]]:
                        q[i, k] = max(q[i, k] - 1, 0)

    def step_cols(q, v, cnt, t):                # eqs.(3)(1)(2) of this rank's columns at step t -> crossers
        cand = []
        for k in range(len(cols)):
            if cnt[k] > 0:
                cnt[k] -= 1
                continue
            S = int(sum(q[i, k] for i in range(N_IN) if S_in[t][i]))
            v[k] = lif(v[k], S)
            if v[k] > Vth:
                cand.append(k)
        return cand

    q = q0[:, lo:hi].astype(np.int64).copy()
    v, cnt, lpost = [Vinit] * len(cols), [0] * len(cols), [-1] * len(cols)
    raster = np.zeros((T, N_EXC), bool)
    NONE = 2 ** 31 - 1
    k0, epochs = 0, 0
    while k0 < T:
        # speculation on copies: run ahead to this rank's first crossing
        qs, vs, cs_ = q.copy(), list(v), list(cnt)
        c_loc, key = NONE, 0
        for t in range(k0, T):
            cand = step_cols(qs, vs, cs_, t)
            if cand:
                c_loc = t
                key = max(((vs[k] + (1 << 31)) << 32) | (0xFFFFFFFF - cols[k]) for k in cand)
                break
            ltd(qs, lpost, t)
        # the 16-byte summary, gathered from every rank; the same reduction everywhere
        summ = [torch.zeros(3, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(summ, torch.tensor([c_loc, key >> 32, key & 0xFFFFFFFF], dtype=torch.int64))
        tstar = min(int(x[0]) for x in summ)
        event = tstar != NONE
        t_end = tstar if event else T - 1
        W = -1
        if event:
            K = max((int(x[1]) << 32) | int(x[2]) for x in summ if int(x[0]) == tstar)
            W = 0xFFFFFFFF - (K & 0xFFFFFFFF)
        # commit [k0, t_end] from the epoch start (no crossing anywhere before t*)
        for t in range(k0, t_end + 1):
            step_cols(q, v, cnt, t)
            if event and t == tstar:
                for k, j in enumerate(cols):
                    v[k] = Vreset
                    if j == W:
                        cnt[k] = p["t_ref_steps"]
                        raster[t, j] = True
                    else:
                        cnt[k] = max(cnt[k], p["t_inh_steps"])
            ltd(q, lpost, t)
            if event and t == tstar and lo <= W < hi:
                kW = W - lo
                for i in range(N_IN):
                    lp = max((tt for tt in range(t + 1) if S_in[tt][i]), default=-1)   # last_pre incl. t* (R14)
                    if lp >= 0 and t - lp < len(pot) and _draw(seed, t, W, i >> 2, 3, i & 3) < pot[t - lp]:
                        q[i, kW] = min(q[i, kW] + 1, qmax)
                lpost[kW] = t
        k0 = t_end + 1
        epochs += 1
    np.save(os.path.join(out_dir, f"q{rank}.npy"), q)
    np.save(os.path.join(out_dir, f"r{rank}.npy"), raster[:, lo:hi])
    np.save(os.path.join(out_dir, f"e{rank}.npy"), np.array([epochs]))
    dist.barrier()
    dist.destroy_process_group()


def test_per_epoch_summary_protocol_matches_oracle(tmp_path):
    # t_ref > t_inh and two strong columns on different ranks: the winner alternates across the ranks
    p = O.params("8b", membrane_mode=1, wta_mode=0, inh_mode=0, f_min_hz=40.0, f_max_hz=400.0, v_spike=12.0,
                 t_ref_steps=10, t_inh_steps=2, init_seed=23)
    net = O.OracleNet(N_IN, N_EXC, BITS, p)
    rng = np.random.default_rng(0)
    q0 = rng.integers(0, 200, size=(N_IN, N_EXC)).astype(np.uint8)
    q0[:, 3] = rng.integers(200, 256, size=N_IN)
    q0[:, 14] = rng.integers(200, 256, size=N_IN)
    net.set_weights(q0)
    image = (np.arange(N_IN) * 53 % 256).astype(np.uint8)
    seed = 777
    net.present(image, T, seed)
    world = 2
    port = 29700 + (os.getpid() % 1000)
    mp.spawn(epoch_worker, args=(world, port, p, q0, image, seed, str(tmp_path)), nprocs=world, join=True)
    q = np.concatenate([np.load(tmp_path / f"q{r}.npy") for r in range(world)], axis=1)
    r = np.concatenate([np.load(tmp_path / f"r{r}.npy") for r in range(world)], axis=1)
    ref = O.unpack_bits(net.spikes(), N_EXC)
    assert ref.sum() >= 4, "the configuration must spike several times"
    assert ref[:, :N_EXC // 2].any() and ref[:, N_EXC // 2:].any(), "winners on both ranks"
    assert np.array_equal(r, ref)
    assert np.array_equal(q.astype(np.uint8), net.weights())
    # one exchange per post spike (+ the last, spike-free epoch), not one per step
    assert int(np.load(tmp_path / "e0.npy")[0]) <= int(ref.sum()) + 1 < T
