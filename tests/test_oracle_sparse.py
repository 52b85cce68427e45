"""Pins of the oracle's NEXT-4 function (Fig. 4 workload: 10^3 LIF neurons, 10^4 synapses, no learning;
P:92 §IV-A; readings DESIGN.md R24-R26).  No GPU."""
import math

import numpy as np
import pytest

from oracle import oracle as O
import synthdata


def _column_graph(W):
    """Feed-forward CSR graph with one synapse per (input i, neuron j) carrying code W[i, j] (no recurrence)."""
    n_in, n = W.shape
    off = np.zeros(n_in + n + 1, np.int32)
    off[1:n_in + 1] = np.arange(1, n_in + 1) * n
    off[n_in + 1:] = n_in * n
    return off, np.tile(np.arange(n, dtype=np.uint16), n_in), W.reshape(-1).astype(np.uint8)


@pytest.mark.parametrize("mode", [0, 1])
def test_sparse_equals_pinned_single_neuron_path(mode):
    """A neuron fed by a full column of synapses is the dense path's neuron: with one neuron the WTA of
    the pinned learning loop never acts on anyone else, so its raster with frozen weights (R21) must
    equal the sparse run's raster, neuron by neuron (eq.(3) over the same codes, same encoder draws)."""
    p = O.params("8b", membrane_mode=mode, v_spike=3.0, f_min_hz=5.0, f_max_hz=78.0)
    rng = np.random.default_rng(3)
    W = rng.integers(0, 256, size=(784, 3)).astype(np.uint8)
    imgs = synthdata.images(2, "mnist")
    seeds = synthdata.seeds(2, base_seed=4)
    net = O.OracleNet(784, 3, 8, p)
    counts, raster = net.sparse_run(3, *_column_graph(W), imgs, 120, seeds, raster=True)
    assert counts.sum() > 0
    for j in range(3):
        one = O.OracleNet(784, 1, 8, p)
        one.set_weights(W[:, j:j + 1])
        for k in range(2):
            one.present_ex(imgs[k], 120, int(seeds[k]), O.ORACLE_NO_LEARN)
            ref = O.unpack_bits(one.spikes(), 1)[:, 0]
            got = O.unpack_bits(raster[k], 3)[:, j]
            assert np.array_equal(ref, got)
            assert counts[k, j] == ref.sum()


def _k_first(I, v0, p=O.BASE):
    a, b, c, vth, dt = p["a"], p["b"], p["c"], p["v_th"], p["dt_ms"]
    lam, vinf = 1.0 + b * dt, -(a + c * I) / b
    return math.floor(math.log((vinf - vth) / (vinf - v0)) / math.log(lam)) + 1


@pytest.mark.parametrize("mode", [0, 1])
def test_recurrent_one_step_delay(mode):
    """R25: a neuron's spike reaches its targets one step later.  Neuron 0: saturating input (p = 1) with
    I = 784/256 per step -> spikes at k(I,-70)-1 and every t_ref + k(I, v_reset) steps after (closed form).
    Neuron 1: no input except a 255-code synapse from neuron 0 (I = 63.75 mV-units: one step lifts it over
    threshold from any v >= v_reset) -> its raster is neuron 0's shifted by exactly one step."""
    p = O.params("8b", membrane_mode=mode, v_spike=64.0, f_min_hz=1000.0, f_max_hz=1000.0)
    n_in = 784
    off = np.zeros(n_in + 2 + 1, np.int32)
    off[1:n_in + 1] = np.arange(1, n_in + 1)          # input i -> neuron 0 (one synapse each)
    off[n_in + 1] = n_in + 1                           # neuron 0 -> neuron 1
    off[n_in + 2] = n_in + 1
    tgt = np.concatenate([np.zeros(n_in, np.uint16), np.array([1], np.uint16)])
    q = np.zeros(n_in + 1, np.uint8)
    q[:12] = 1                                         # 12 always-on inputs of code 1: I = 64 * 12 / 256 = 3.0
    q[n_in] = 255                                      # neuron 0 -> neuron 1: I = 63.75
    net = O.OracleNet(n_in, 2, 8, p)
    counts, raster = net.sparse_run(2, off, tgt, q, np.full((1, n_in), 9, np.uint8), 200, [5], raster=True)
    r = O.unpack_bits(raster[0], 2)
    s0 = np.nonzero(r[:, 0])[0]
    s1 = np.nonzero(r[:, 1])[0]
    first, period = _k_first(3.0, -70.0) - 1, p["t_ref_steps"] + _k_first(3.0, p["v_reset"])
    assert s0.tolist() == list(range(first, 200, period))
    assert s1.tolist() == [s + 1 for s in s0 if s + 1 < 200]


def test_sparse_invariants():
    p = O.params("4b", membrane_mode=1, v_spike=40.0, f_min_hz=5.0, f_max_hz=78.0, t_ref_steps=3)
    off, tgt, q = synthdata.sparse_graph(784, 300, 3000, bits=4, seed=7)
    isolated = np.setdiff1d(np.arange(300), tgt)
    net = O.OracleNet(784, 300, 4, p)
    counts, raster = net.sparse_run(300, off, tgt, q, synthdata.images(2, "fashion"), 150, [1, 2], raster=True)
    assert counts.sum() > 0
    assert (counts[:, isolated] == 0).all()                   # no synapse in -> never spikes (i_ext = 0)
    r = O.unpack_bits(raster.reshape(-1, raster.shape[-1]), 300).reshape(2, 150, -1)[:, :, :300]
    for k in range(2):
        for j in np.nonzero(counts[k])[0]:
            st = np.nonzero(r[k, :, j])[0]
            assert (np.diff(st) >= p["t_ref_steps"] + 1).all()   # refractory period (R6)
    assert np.array_equal(r.sum(axis=1), counts)


def test_sparse_rejects_bad_graph():
    net = O.OracleNet(784, 10, 4, O.params("4b"))
    off, tgt, q = synthdata.sparse_graph(784, 10, 100, bits=4)
    bad = q.copy(); bad[0] = 16
    with pytest.raises(O.OracleError):
        net.sparse_run(10, off, tgt, bad, synthdata.images(1), 5, [1])
    badt = tgt.copy(); badt[0] = 10
    with pytest.raises(O.OracleError):
        net.sparse_run(10, off, badt, q, synthdata.images(1), 5, [1])
