"""Column-sharded per-step engine (NEXT-2 at C4 scale) against the unsharded
oracle (needs a B200).  On the per-step engine every step's WTA summary of each shard's cluster (best key for
HARD, spiker count for LAYER) goes to every shard's device-memory mailbox and every shard applies the same
reduction.  This is what lets a 784 -> 6400 network with 16-bit codes (10 MB, R27) or binary32 conductances
(20 MB, R28) learn: 4 / 7 clusters of <= 16 CTAs on one B200, presented in ONE snn_present_many launch.
The union of the shards must equal the oracle: codes / conductances, rasters, per-image spike counts, state
and counters (membranes within 1e-5 relative in fp32 mode)."""
import numpy as np
import pytest

import synthdata
from oracle import oracle as O

from test_gpu_sharding import _compare

pytestmark = pytest.mark.gpu


def _step_shards(n_in, n_exc, bits, p, world):
    import paper_conf_date_shelm19_b200 as P
    sh = [P.Network(n_in, n_exc, bits, P.params_from_dict(p, engine=1), shard=(r, world)) for r in range(world)]
    assert all(s.info()["engine"] == 1 for s in sh)
    P.link_shards(sh)
    return sh


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("wta,stdp", [(0, 0), (1, 0), (0, 1)])
def test_step_sharded_784x400_8bit(gpu, world, wta, stdp):
    p = O.params("8b", wta_mode=wta, stdp_mode=stdp, membrane_mode=1, init_seed=3)
    sh = _step_shards(784, 400, 8, p, world)
    o = O.OracleNet(784, 400, 8, p)
    _compare(sh, o, synthdata.images(2, "mnist", start=300), 150, synthdata.seeds(2, base_seed=41), 784, 400, 1)
    assert int(o.stats()[1]) > 0


def test_step_sharded_16bit_784x800(gpu):
    p = O.params("16b", rounding=2, membrane_mode=0, init_seed=4)
    sh = _step_shards(784, 800, 16, p, 2)
    o = O.OracleNet(784, 800, 16, p)
    _compare(sh, o, synthdata.images(2, "fashion", start=10), 120, synthdata.seeds(2, base_seed=42), 784, 800, 0)


def test_step_sharded_16bit_C4_784x6400(gpu):
    """NEXT-2 at the C4 network: 784 -> 6400 with 16-bit codes (10 MB) as 4 shards x 16 CTAs."""
    import paper_conf_date_shelm19_b200 as P
    p = O.params("16b", rounding=2, membrane_mode=1, init_seed=5)
    with pytest.raises(P.SnnError):                  # one cluster cannot hold it
        P.Network(784, 6400, 16, P.params_from_dict(p))
    sh = _step_shards(784, 6400, 16, p, 4)
    o = O.OracleNet(784, 6400, 16, p)
    _compare(sh, o, synthdata.images(1, "fashion", start=20), 60, synthdata.seeds(1, base_seed=43), 784, 6400, 1)
    assert int(o.stats()[1]) > 0


def test_step_sharded_fp32_C4_784x6400(gpu):
    """NEXT-2 at the C4 network with binary32 conductances (20 MB, R28) as 7 shards of 15-16 CTAs (7 clusters of
    16 CTAs is what a B200's GPCs hold at once)."""
    p = O.params("16b", init_seed=6)
    sh = _step_shards(784, 6400, 32, p, 7)
    o = O.OracleNet(784, 6400, 32, p)
    _compare(sh, o, synthdata.images(1, "fashion", start=21), 60, synthdata.seeds(1, base_seed=44), 784, 6400, 0)
    assert int(o.stats()[1]) > 0


def test_step_sharded_fp32_deterministic_layer(gpu):
    p = O.params("16b", stdp_mode=1, wta_mode=1, init_seed=7)
    sh = _step_shards(784, 640, 32, p, 3)
    o = O.OracleNet(784, 640, 32, p)
    _compare(sh, o, synthdata.images(2, "mnist", start=30), 120, synthdata.seeds(2, base_seed=45), 784, 640, 0)


def _wide_fuzz_case(k):
    rng = np.random.default_rng(7000 + k)
    bits = int(rng.choice([16, 32]))
    world = int(rng.choice([1, 1, 2, 3]))
    n_exc = int(rng.choice([33, 64, 100, 200, 320]))
    n_exc = max(n_exc, 32 * world)
    fmin, fmax = [(1.0, 22.0), (5.0, 78.0)][int(rng.integers(2))]
    kw = dict(init_seed=int(rng.integers(1, 99)), wta_mode=int(rng.random() < 0.4), stdp_mode=int(rng.random() < 0.4),
              inh_mode=int(rng.random() < 0.25), f_min_hz=fmin, f_max_hz=fmax,
              t_ref_steps=int(rng.choice([1, 5, 10])), t_inh_steps=int(rng.choice([3, 10])),
              v_spike=float(rng.choice([1.0, 2.0, 3.0])))
    if bits == 16:
        kw.update(membrane_mode=int(rng.integers(2)), rounding=int(rng.integers(3)), frac_bits=int(rng.choice([0, 15])))
    p = O.params(str(rng.choice(["16b", "hf"])), **kw)
    return p, bits, world, n_exc, int(rng.choice([60, 150])), str(rng.choice(["mnist", "fashion"])), int(rng.integers(5000))


@pytest.mark.parametrize("k", range(16))
def test_wide_step_fuzz_vs_oracle(gpu, k):
    """Randomised 16-bit (R27) and binary32 (R28) networks on the per-step engine, unsharded and column-sharded
    (world 1-3): widths, column counts, both STDP arms, HARD/LAYER, RESET/HOLD, rates, refractory / inhibition
    lengths, current scale, membrane mode, rounding, Q1.15; 2 images against the oracle."""
    import paper_conf_date_shelm19_b200 as P
    p, bits, world, n_exc, T, kind, start = _wide_fuzz_case(k)
    o = O.OracleNet(784, n_exc, bits, p)
    imgs, seeds = synthdata.images(2, kind, start=start), synthdata.seeds(2, base_seed=k + 3)
    mode = p["membrane_mode"]
    if world == 1:
        g = P.Network(784, n_exc, bits, P.params_from_dict(p))
        for x, s in zip(imgs, seeds):
            g.present(x, T, int(s))
            o.present(x, T, int(s))
            assert np.array_equal(g.spikes(), o.spikes()), "raster"
            assert np.array_equal(g.weights(), o.weights()), "codes"
            sg, so = O.unpack_state(g.state(), 784, n_exc), O.unpack_state(o.state(), 784, n_exc)
            for key in ("cnt", "last_post", "last_pre"):
                assert np.array_equal(sg[key], so[key]), key
            if mode == 1:
                assert np.array_equal(sg["v"], so["v"])
            else:
                np.testing.assert_allclose(sg["v"], so["v"], rtol=1e-5, atol=0)
    else:
        sh = _step_shards(784, n_exc, bits, p, world)
        _compare(sh, o, imgs, T, seeds, 784, n_exc, mode)


@pytest.mark.parametrize("bits,world", [(16, 4), (32, 7)])
def test_sharded_wide_C4_inference(gpu, bits, world):
    """NEXT-1 on the C4 network at 16 bits / binary32 (column-sharded over 4 / 7 clusters): snn_infer_many runs
    the shards in one launch with frozen weights; the concatenated per-neuron counts equal the oracle's inference."""
    import paper_conf_date_shelm19_b200 as P
    p = O.params("16b", init_seed=15, f_min_hz=5.0, f_max_hz=78.0, **({"rounding": 2} if bits == 16 else {}))
    sh = _step_shards(784, 6400, bits, p, world)
    o = O.OracleNet(784, 6400, bits, p)
    imgs, seeds = synthdata.images(2, "fashion", start=77), synthdata.seeds(2, base_seed=78)
    w0 = [s.weights().copy() for s in sh]
    outs = P.infer_many(sh, [imgs] * world, 60, [seeds] * world)
    want = o.infer(imgs, 60, seeds)
    assert np.array_equal(np.concatenate(outs, axis=1), want)
    assert int(want.sum()) > 0
    assert all(np.array_equal(s.weights().view(np.uint8), w.view(np.uint8)) for s, w in zip(sh, w0))
    with pytest.raises(P.SnnError):                  # the world must be complete
        P.infer_many(sh[:1], [imgs], 60, [seeds])
