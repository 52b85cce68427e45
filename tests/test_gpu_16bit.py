"""NEXT-2 GPU <-> oracle parity: 16-bit conductance codes ("For 16-bit ... after floating point
calculation of change in conductance dG, the result is rounded"; Table I "16 bit" / "high frequency" rows,
P:103; reading DESIGN.md R27).  Codes, rasters, timers, counters bit-exact; membranes bit-exact in Q15.16
and within 1e-5 relative in fp32 (same bar as tests/test_gpu_parity.py)."""
import numpy as np
import pytest

import synthdata
from oracle import oracle as O

pytestmark = pytest.mark.gpu


def _pair(n_in, n_exc, p):
    import paper_conf_date_shelm19_b200 as P
    return P.Network(n_in, n_exc, 16, P.params_from_dict(p)), O.OracleNet(n_in, n_exc, 16, p)


def _compare(g, o, imgs, T, seeds, n_in, n_exc, mode):
    for img, sd in zip(imgs, seeds):
        g.reset_stats()
        g.present(img, T, int(sd))
        o.present(img, T, int(sd))
        assert np.array_equal(g.spikes(), o.spikes()), "raster"
        assert np.array_equal(g.weights(), o.weights()), "codes"
        assert np.array_equal(g.stats()[:6], o.stats()[:6]), "counters"
        sg, so = O.unpack_state(g.state(), n_in, n_exc), O.unpack_state(o.state(), n_in, n_exc)
        for k in ("cnt", "last_post", "last_pre"):
            assert np.array_equal(sg[k], so[k]), k
        if mode == 1:
            assert np.array_equal(sg["v"], so["v"])
        else:
            np.testing.assert_allclose(sg["v"], so["v"], rtol=1e-5, atol=0)


def test_16bit_init_and_roundtrip(gpu):
    p = O.params("16b", init_seed=7)
    g, o = _pair(784, 100, p)
    w = g.weights()
    assert w.dtype == np.uint16 and int(w.max()) > 255
    assert np.array_equal(w, o.weights())
    rng = np.random.default_rng(1)
    c = rng.integers(0, 65536, size=(784, 100)).astype(np.uint16)
    g.set_weights(c)
    assert np.array_equal(g.weights(), c)


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("rounding", [0, 1, 2])
def test_16bit_stochastic_c1(gpu, mode, rounding):
    """784 -> 100, Table I "16 bit" row (gamma 0.9), stochastic STDP with eq.(4)/(5) steps, 4 images."""
    p = O.params("16b", membrane_mode=mode, rounding=rounding, init_seed=3)
    g, o = _pair(784, 100, p)
    imgs = synthdata.images(4, "mnist", start=30)
    seeds = synthdata.seeds(4, base_seed=12)
    _compare(g, o, imgs, 100, seeds, 784, 100, mode)
    assert int(o.stats()[3]) + int(o.stats()[5]) > 0


@pytest.mark.parametrize("stdp,wta", [(0, 1), (1, 0), (1, 1)])
def test_16bit_c2_shapes(gpu, stdp, wta):
    """784 -> 400 (the C2 shape: 627 KB of 16-bit codes over a cluster), LAYER / HARD WTA, both arms."""
    p = O.params("16b", stdp_mode=stdp, wta_mode=wta, rounding=2, membrane_mode=1, init_seed=5)
    g, o = _pair(784, 400, p)
    imgs = synthdata.images(2, "mnist", start=70)
    seeds = synthdata.seeds(2, base_seed=2)
    _compare(g, o, imgs, 120, seeds, 784, 400, 1)


def test_16bit_high_frequency_row(gpu):
    """Table I "high frequency" row (5-78 Hz, tau_pot 80, tau_dep 5) at 16 bits, T = 100."""
    p = O.params("hf", membrane_mode=0, rounding=1, init_seed=8)
    g, o = _pair(784, 64, p)
    imgs = synthdata.images(3, "mnist", start=5)
    seeds = synthdata.seeds(3, base_seed=5)
    _compare(g, o, imgs, 100, seeds, 784, 64, 0)


def test_16bit_q115_frac15(gpu):
    """Q1.15 labels: frac_bits = 15 -> q_max = G_max * 2^15 = 32768 (R9)."""
    p = O.params("16b", frac_bits=15, membrane_mode=1, init_seed=2)
    g, o = _pair(784, 50, p)
    assert o.q_max == 32768
    imgs = synthdata.images(2, "mnist", start=11)
    seeds = synthdata.seeds(2, base_seed=9)
    _compare(g, o, imgs, 100, seeds, 784, 50, 1)


def test_16bit_rejections(gpu):
    import paper_conf_date_shelm19_b200 as P
    g = P.Network(784, 64, 16, P.preset("16b"))
    assert g.info()["engine"] == 1                       # per-step engine selected automatically
    assert g.infer(synthdata.images(1), 10, synthdata.seeds(1)).shape == (1, 64)   # per-step engine inference
    sh = P.Network(784, 640, 16, P.preset("16b"), shard=(0, 2))   # shards run on the per-step engine
    assert sh.info()["engine"] == 1 and sh.info()["world"] == 2
    with pytest.raises(P.SnnError):                      # inference runs on unsharded handles
        sh.infer(synthdata.images(1), 10, synthdata.seeds(1))


def test_table2_grid_ensemble_mixed_widths(gpu):
    """The Table II grid (precisions x rounding x rule) as ONE snn_present_many launch on the per-step
    engine (same cluster shape for every width, 16-bit included): every network bit-exact with its oracle."""
    import paper_conf_date_shelm19_b200 as P
    rows = {2: "2b", 4: "4b", 8: "8b", 16: "16b"}
    nets, oracles, imgs, seeds = [], [], [], []
    k = 0
    for bits in (2, 4, 8, 16):
        for rounding in (0, 2):
            for stdp in (0, 1):
                p = O.params(rows[bits], stdp_mode=stdp, rounding=rounding, membrane_mode=1, init_seed=1 + k,
                             cluster_size=4)
                nets.append(P.Network(784, 128, bits, P.params_from_dict(p, engine=1)))
                oracles.append(O.OracleNet(784, 128, bits, p))
                imgs.append(synthdata.images(2, "mnist", start=20 * k))
                seeds.append(synthdata.seeds(2, base_seed=300 + k))
                k += 1
    P.present_many(nets, imgs, 100, seeds)
    for g, o, im, sd in zip(nets, oracles, imgs, seeds):
        for x, s in zip(im, sd):
            o.present(x, 100, int(s))
        assert np.array_equal(g.weights(), o.weights())
        assert np.array_equal(g.spikes(), o.spikes())
