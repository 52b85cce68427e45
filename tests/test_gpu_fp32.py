"""NEXT-2 GPU <-> oracle parity: 32-bit floating-point conductance ("32-bit floating-point (accuracy
96.1%)"; "For 16-bit and 32-bit learning, after floating point calculation of change in conductance dG,
the result is rounded to a value that can be represented in the current bit width"; reading DESIGN.md R28).

Both sides execute the same sequence of IEEE-rounded operations (binary32 sums in ascending row order, the
fp32 LIF recipe, binary64 eqs.(4)(5) through R28's exp recipe, one rounding to binary32 per event), so
conductances, rasters, timers and counters are compared bit for bit; membranes within 1e-5 relative (the
north_star's fp32 bar; bit-exact in practice)."""
import numpy as np
import pytest

import synthdata
from oracle import oracle as O

pytestmark = pytest.mark.gpu


def _pair(n_in, n_exc, p):
    import paper_conf_date_shelm19_b200 as P
    return P.Network(n_in, n_exc, 32, P.params_from_dict(p)), O.OracleNet(n_in, n_exc, 32, p)


def _compare_state(g, o, n_in, n_exc):
    assert np.array_equal(g.spikes(), o.spikes()), "raster"
    gw, ow = g.weights(), o.weights()
    assert gw.dtype == np.float32
    bad = np.argwhere(gw.view(np.uint32) != ow.view(np.uint32))
    assert bad.size == 0, f"{len(bad)} conductances differ, first {bad[:3].tolist()}: {gw[tuple(bad[0])]} vs {ow[tuple(bad[0])]}"
    assert np.array_equal(g.stats()[:6], o.stats()[:6]), "counters"
    sg, so = O.unpack_state(g.state(), n_in, n_exc), O.unpack_state(o.state(), n_in, n_exc)
    for k in ("cnt", "last_post", "last_pre"):
        assert np.array_equal(sg[k], so[k]), k
    np.testing.assert_allclose(sg["v"], so["v"], rtol=1e-5, atol=0)


def _compare(g, o, imgs, T, seeds, n_in, n_exc):
    for img, sd in zip(imgs, seeds):
        g.reset_stats()
        g.present(img, T, int(sd))
        o.present(img, T, int(sd))
        _compare_state(g, o, n_in, n_exc)


def test_fp32_init_and_roundtrip(gpu):
    import paper_conf_date_shelm19_b200 as P
    for g_max in (1.0, 0.75):
        p = O.params("16b", init_seed=7, g_max=g_max)
        g, o = _pair(784, 100, p)
        w = g.weights()
        assert w.dtype == np.float32 and w.max() < g_max and w.min() >= 0.0
        assert np.array_equal(w.view(np.uint32), o.weights().view(np.uint32))
    rng = np.random.default_rng(1)
    c = (rng.random((784, 100)) * 0.75).astype(np.float32)
    g.set_weights(c)
    assert np.array_equal(g.weights(), c)
    for bad in (0.7501, -1e-7, np.nan, np.inf):
        c2 = c.copy()
        c2[3, 4] = bad
        with pytest.raises(P.SnnError):
            g.set_weights(c2)
    assert np.array_equal(g.weights(), c)


@pytest.mark.parametrize("wta", [0, 1])
def test_fp32_stochastic_c1(gpu, wta):
    """784 -> 100, Table I "16 bit" row (gamma 0.9): eqs.(6)(7)-gated events of eq.(4)/(5) size, 4 images."""
    p = O.params("16b", wta_mode=wta, init_seed=3)
    g, o = _pair(784, 100, p)
    _compare(g, o, synthdata.images(4, "mnist", start=30), 100, synthdata.seeds(4, base_seed=12), 784, 100)
    assert int(o.stats()[3]) + int(o.stats()[5]) > 0


@pytest.mark.parametrize("wta", [0, 1])
def test_fp32_deterministic_c1(gpu, wta):
    """Deterministic arm (R16 window, eqs.(4)(5) magnitudes in binary32): the floating-point baseline of P:82."""
    p = O.params("16b", stdp_mode=1, wta_mode=wta, init_seed=4)
    g, o = _pair(784, 100, p)
    _compare(g, o, synthdata.images(3, "mnist", start=40), 150, synthdata.seeds(3, base_seed=13), 784, 100)
    assert int(o.stats()[1]) > 0


@pytest.mark.parametrize("stdp,wta", [(0, 0), (0, 1), (1, 1)])
def test_fp32_c2_shape(gpu, stdp, wta):
    """784 -> 400 (C2's network: 1.25 MB of binary32 conductance over one cluster), 350-step presentations."""
    p = O.params("16b", stdp_mode=stdp, wta_mode=wta, init_seed=5)
    g, o = _pair(784, 400, p)
    assert g.info()["cluster_size"] >= 7
    _compare(g, o, synthdata.images(2, "mnist", start=70), 350, synthdata.seeds(2, base_seed=2), 784, 400)


def test_fp32_high_frequency_row(gpu):
    """Table I "high frequency" row (5-78 Hz, tau_pot 80, tau_dep 5), T = 100, fashion-shaped input."""
    p = O.params("hf", init_seed=8)
    g, o = _pair(784, 64, p)
    _compare(g, o, synthdata.images(3, "fashion", start=5), 100, synthdata.seeds(3, base_seed=5), 784, 64)


def test_fp32_ragged_small(gpu):
    """Ragged shapes: 37 columns (a partial 32-column group), 50 inputs (a partial input word)."""
    p = O.params("16b", f_min_hz=20.0, f_max_hz=200.0, init_seed=6)
    g, o = _pair(50, 37, p)
    imgs = synthdata.images(3, "fashion", start=2)[:, :50]
    _compare(g, o, imgs, 80, synthdata.seeds(3, base_seed=21), 50, 37)


def test_fp32_batch_matches_sequential_oracle(gpu):
    """One snn_present_batch launch of 6 images (weights resident on chip across images) against the oracle
    presenting them one by one: final conductances, per-image spike counts, last raster and state."""
    import paper_conf_date_shelm19_b200 as P
    p = O.params("16b", init_seed=9)
    g, o = _pair(784, 128, p)
    imgs = synthdata.images(6, "mnist", start=90)
    seeds = synthdata.seeds(6, base_seed=31)
    counts = np.zeros(6, np.int32)
    g.present_batch(imgs, 100, seeds, spike_counts=counts)
    want = []
    for img, sd in zip(imgs, seeds):
        o.present(img, 100, int(sd))
        want.append(int(O.unpack_bits(o.spikes(), 128).sum()))
    assert counts.tolist() == want
    assert np.array_equal(g.weights().view(np.uint32), o.weights().view(np.uint32))
    assert np.array_equal(g.spikes(), o.spikes())
    sg, so = O.unpack_state(g.state(), 784, 128), O.unpack_state(o.state(), 784, 128)
    for k in ("cnt", "last_post", "last_pre"):
        assert np.array_equal(sg[k], so[k]), k


def test_fp32_rejections(gpu):
    import paper_conf_date_shelm19_b200 as P
    g = P.Network(784, 64, 32, P.preset("16b"))
    assert g.info()["engine"] == 1                       # per-step engine selected automatically
    assert g.infer(synthdata.images(1), 10, synthdata.seeds(1)).shape == (1, 64)   # per-step engine inference
    sh = P.Network(784, 640, 32, P.preset("16b"), shard=(0, 2))   # shards run on the per-step engine
    assert sh.info()["engine"] == 1 and sh.info()["world"] == 2
    with pytest.raises(P.SnnError):                      # inference runs on unsharded handles
        sh.infer(synthdata.images(1), 10, synthdata.seeds(1))
    with pytest.raises(P.SnnError):
        P.Network(784, 64, 32, P.params_from_dict(O.params("16b", membrane_mode=1)))
    with pytest.raises(P.SnnError):
        P.Network(784, 64, 32, P.params_from_dict(O.params("16b", rounding=2)))
    with pytest.raises(P.SnnError):                      # 5 MB of binary32 > one cluster's shared memory
        P.Network(784, 1600, 32, P.preset("16b"))


def test_fp32_stepwise_keep_state_and_reseed(gpu):
    """North-star protocol at 32 bits: one step per call with SNN_KEEP_STATE (t0 = t); after every step the state
    and the conductances equal the oracle's; at t = 40 the GPU is reseeded from the oracle (state + G) and goes on."""
    import paper_conf_date_shelm19_b200 as P
    p = O.params("16b", init_seed=8, f_min_hz=5.0, f_max_hz=78.0)
    g, o = _pair(784, 64, p)
    img = synthdata.images(1, "mnist", start=4)[0]
    for t in range(80):
        o.present_ex(img, 1, 21, flags=O.ORACLE_KEEP_STATE if t else 0, t0=t)
        g.reset_stats()                                  # the library's counters accumulate across calls
        g.present_ex(img, 1, 21, flags=(P.SNN_KEEP_STATE if t else 0), t0=t)
        _compare_state(g, o, 784, 64)
        if t == 40:
            g.set_state(o.state())
            g.set_weights(o.weights())
    assert int(O.unpack_bits(o.spikes(), 64).sum()) >= 0


def test_fp32_raster_input_forced_ltp_ltd(gpu):
    """Encoder bypass (SNN_RASTER_INPUT) with forced post spikes: every LTP / LTD event of the binary32 arm (eq.(4)
    / eq.(5) magnitudes) and its counters equal the oracle's."""
    p = O.params("16b", i_ext=60.0, v_spike=1e-9, t_ref_steps=7, gamma_pot=0.9, gamma_dep=0.9)
    g, o = _pair(784, 3, p)
    rng = np.random.default_rng(3)
    raster = rng.integers(0, 2 ** 32, size=(40, 25), dtype=np.uint64).astype(np.uint32)
    raster &= rng.integers(0, 2 ** 32, size=(40, 25), dtype=np.uint64).astype(np.uint32)
    raster[:, -1] &= 0xFFFF
    g.present_raster(raster, 40, 99)
    o.present_raster(raster, 40, 99)
    _compare_state(g, o, 784, 3)
    assert o.stats()[3] > 0 and o.stats()[5] > 0


def test_fp32_and_16bit_ensemble_one_launch(gpu):
    """snn_present_many with binary32 and 16-bit networks side by side on the per-step engine (one launch); each
    network equals its own oracle."""
    import paper_conf_date_shelm19_b200 as P
    specs = [(32, O.params("16b", init_seed=11, cluster_size=2)), (16, O.params("16b", init_seed=12, rounding=2, cluster_size=2)),
             (32, O.params("16b", init_seed=13, stdp_mode=1, cluster_size=2))]
    nets = [P.Network(784, 128, b, P.params_from_dict(p)) for b, p in specs]
    assert {n.info()["cluster_size"] for n in nets} == {2}
    orc = [O.OracleNet(784, 128, b, p) for b, p in specs]
    imgs = [synthdata.images(2, "mnist", start=50 + 7 * k) for k in range(3)]
    seeds = [synthdata.seeds(2, base_seed=60 + k) for k in range(3)]
    P.present_many(nets, imgs, 100, seeds)
    for n, o, im, sd in zip(nets, orc, imgs, seeds):
        for x, s in zip(im, sd):
            o.present(x, 100, int(s))
        assert np.array_equal(n.weights().view(np.uint8), o.weights().view(np.uint8))
        assert np.array_equal(n.spikes(), o.spikes())


@pytest.mark.parametrize("bits,wta", [(32, 0), (32, 1), (16, 0)])
def test_wide_inference_matches_oracle(gpu, bits, wta):
    """NEXT-1 at 16 bits / binary32 (R21 on R27 / R28): snn_infer on the per-step engine with frozen weights equals
    the oracle's inference spike counts for every neuron and image; weights and state are left untouched; labelling
    and the vote (R22, R23) then run on those counts."""
    import paper_conf_date_shelm19_b200 as P
    p = O.params("16b", wta_mode=wta, init_seed=14, f_min_hz=5.0, f_max_hz=78.0,
                 **({"rounding": 2, "membrane_mode": 1} if bits == 16 else {}))
    g = P.Network(784, 100, bits, P.params_from_dict(p))
    o = O.OracleNet(784, 100, bits, p)
    learn_imgs, learn_seeds = synthdata.images(2, "mnist", start=300), synthdata.seeds(2, base_seed=70)
    for x, s in zip(learn_imgs, learn_seeds):           # some learning first, identical on both sides
        g.present(x, 100, int(s))
        o.present(x, 100, int(s))
    w0, st0 = g.weights().copy(), g.state().copy()
    imgs, seeds = synthdata.images(6, "mnist", start=310), synthdata.seeds(6, base_seed=71)
    c = g.infer(imgs, 120, seeds)
    want = o.infer(imgs, 120, seeds)
    assert np.array_equal(c, want)
    assert int(want.sum()) > 0
    assert np.array_equal(g.weights().view(np.uint8), w0.view(np.uint8)) and np.array_equal(g.state(), st0)
    classes = synthdata.labels(6)
    lab = g.label(c, classes, 10)
    assert np.array_equal(lab, O.label(want, classes, 10))
    assert np.array_equal(g.classify(c, lab, 10), O.classify(want, lab, 10))
