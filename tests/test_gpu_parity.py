"""GPU <-> oracle parity (needs a B200).  Every comparison goes through the C ABI (libsnn_b200.so)
on one side and the CPU oracle on the other, on the same seeded synthetic inputs.

Bar: integer work -- input rasters, output rasters, conductance codes, spike
timers, refractory counters, counters -- bit-exact; membrane potentials bit-exact in the
Q15.16 mode and within 1e-5 relative per step in the fp32 mode (the recipes are identical
fmaf sequences, so in practice they are bit-exact too; the tolerance is what is asserted)."""
import numpy as np
import pytest

import synthdata
from oracle import oracle as O

pytestmark = pytest.mark.gpu


# SNN_ENGINE_EVENT (event-driven epochs; the lean kernel where HARD + RESET + stochastic applies),
# SNN_ENGINE_STEP (per-step exchange), SNN_ENGINE_EVENT_GENERAL (the general event kernel everywhere)
ENGINES = [0, 1, 2]


def _pair(n_in, n_exc, bits, p, engine=0):
    import paper_conf_date_shelm19_b200 as P
    g = P.Network(n_in, n_exc, bits, P.params_from_dict(p, engine=engine))
    o = O.OracleNet(n_in, n_exc, bits, p)
    return g, o


def _assert_state_equal(g, o, n_in, n_exc, mode):
    sg = O.unpack_state(g.state(), n_in, n_exc)
    so = O.unpack_state(o.state(), n_in, n_exc)
    for k in ("n_in", "n_exc", "t_next", "membrane_mode"):
        assert sg[k] == so[k], k
    for k in ("cnt", "last_post", "last_pre"):
        assert np.array_equal(sg[k], so[k]), k
    if mode == 1:
        assert np.array_equal(sg["v"], so["v"])
    else:
        np.testing.assert_allclose(sg["v"], so["v"], rtol=1e-5, atol=0)


def _compare_presentations(g, o, images, T, seeds, n_in, n_exc, mode, record=True):
    import paper_conf_date_shelm19_b200 as P
    for img, sd in zip(images, seeds):
        g.reset_stats()
        g.present_ex(img, T, int(sd), flags=P.SNN_RECORD_INPUT if record else 0)
        o.present(img, T, int(sd))
        if record:
            assert np.array_equal(g.input_raster(), o.input_raster()), "encoder (a1) raster"
        assert np.array_equal(g.spikes(), o.spikes()), "output raster (a3/a4)"
        assert np.array_equal(g.weights(), o.weights()), "conductance codes (a5)"
        assert np.array_equal(g.stats()[:6], o.stats()[:6]), "counters"
        _assert_state_equal(g, o, n_in, n_exc, mode)


# ------------------------------------------------------------------ a4 init + layout round trips
@pytest.mark.parametrize("bits", [2, 4, 8])
@pytest.mark.parametrize("n_exc,cs", [(100, 0), (33, 0), (400, 2), (1600, 5), (6400, 16)])
def test_initial_weights_bit_exact(gpu, bits, n_exc, cs):
    import paper_conf_date_shelm19_b200 as P
    p = O.params("8b", init_seed=11 + bits, cluster_size=cs)
    if 784 * n_exc * bits / 8 > (cs or 16) * 220 * 1024:
        with pytest.raises(P.SnnError) as e:      # exceeds one cluster's shared memory
            _pair(784, n_exc, bits, p)
        assert e.value.rc == -5
        return
    g, o = _pair(784, n_exc, bits, p)
    assert np.array_equal(g.weights(), o.weights())


def test_set_get_weights_roundtrip(gpu):
    import paper_conf_date_shelm19_b200 as P
    g, _ = _pair(784, 1600, 4, O.params("4b", cluster_size=4))
    w = np.random.default_rng(0).integers(0, 16, size=(784, 1600)).astype(np.uint8)
    g.set_weights(w)
    assert np.array_equal(g.weights(), w)
    with pytest.raises(P.SnnError):
        g.set_weights(np.full((784, 1600), 16, np.uint8))


# ------------------------------------------------------------------ C1: 784 -> 100, 8 bit, T = 100 (configs[0])
@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("engine", ENGINES)
def test_C1_784x100_8bit_20_images(gpu, engine, mode):
    p = O.params("8b", membrane_mode=mode, init_seed=1)
    g, o = _pair(784, 100, 8, p, engine=engine)
    imgs = synthdata.images(20, "mnist")
    seeds = synthdata.seeds(20, base_seed=1)
    _compare_presentations(g, o, imgs, 100, seeds, 784, 100, mode)
    assert o.stats()[1] > 0


@pytest.mark.parametrize("engine", ENGINES)
def test_C1_batch_launch_equals_per_image(gpu, engine):
    """snn_present_batch (one persistent launch, weights resident across images) == the oracle
    presenting the images one by one."""
    p = O.params("8b", membrane_mode=1, init_seed=1)
    g, o = _pair(784, 100, 8, p, engine=engine)
    imgs = synthdata.images(20, "mnist")
    seeds = synthdata.seeds(20, base_seed=1)
    counts = np.zeros(20, np.int32)
    g.present_batch(imgs, 100, seeds, counts)
    oc = []
    for img, sd in zip(imgs, seeds):
        o.present(img, 100, int(sd))
        oc.append(int(O.unpack_bits(o.spikes(), 100).sum()))
    assert counts.tolist() == oc
    assert np.array_equal(g.weights(), o.weights())
    assert np.array_equal(g.spikes(), o.spikes())
    _assert_state_equal(g, o, 784, 100, 1)


# ------------------------------------------------------------------ C2: 784 -> 400 LAYER WTA, stochastic and deterministic arms
@pytest.mark.parametrize("stdp,rounding", [(0, 1), (1, 0), (1, 1), (1, 2)])
@pytest.mark.parametrize("engine", ENGINES)
def test_C2_784x400_layer(gpu, engine, stdp, rounding):
    p = O.params("8b", wta_mode=1, stdp_mode=stdp, rounding=rounding, membrane_mode=1, init_seed=2)
    g, o = _pair(784, 400, 8, p, engine=engine)
    imgs = synthdata.images(3, "mnist", start=100)
    seeds = synthdata.seeds(3, base_seed=2)
    _compare_presentations(g, o, imgs, 350, seeds, 784, 400, 1)
    assert o.stats()[1] > 0


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("engine", ENGINES)
def test_C2_hard_det_fp32(gpu, engine, mode):
    p = O.params("8b", stdp_mode=1, rounding=2, membrane_mode=mode, init_seed=3)
    g, o = _pair(784, 400, 8, p, engine=engine)
    _compare_presentations(g, o, synthdata.images(2, "mnist", start=7), 350, synthdata.seeds(2, 3), 784, 400, mode)


# ------------------------------------------------------------------ C3: 784 -> 1600, 2 bit, rate sweep
@pytest.mark.parametrize("fmin,fmax,T", [(1.0, 22.0, 350), (5.0, 78.0, 100), (5.0, 156.0, 100), (10.0, 312.0, 100)])
@pytest.mark.parametrize("engine", ENGINES)
def test_C3_784x1600_2bit_rate_sweep(gpu, engine, fmin, fmax, T):
    p = O.params("2b", f_min_hz=fmin, f_max_hz=fmax, membrane_mode=1, init_seed=4)
    g, o = _pair(784, 1600, 2, p, engine=engine)
    _compare_presentations(g, o, synthdata.images(2, "mnist", start=3), T, synthdata.seeds(2, 4), 784, 1600, 1)


@pytest.mark.parametrize("cs", [1, 2, 3, 8, 16])
@pytest.mark.parametrize("engine", ENGINES)
def test_cluster_size_invariance(gpu, engine, cs):
    """The same network sliced over 1..16 CTAs gives bit-identical results (global Philox indices)."""
    p = O.params("2b", membrane_mode=1, init_seed=5, cluster_size=cs)
    g, o = _pair(784, 512, 2, p, engine=engine)        # 16 groups of 32 columns: 100 KB on one CTA, 1 group per CTA at 16
    _compare_presentations(g, o, synthdata.images(2, "fashion"), 150, synthdata.seeds(2, 5), 784, 512, 1)


# ------------------------------------------------------------------ C4: 784 -> 6400, 2 bit, fashion (the bench workload)
@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("engine", ENGINES)
def test_C4_784x6400_2bit_full_size(gpu, engine, mode):
    p = O.params("2b", membrane_mode=mode, init_seed=1)
    g, o = _pair(784, 6400, 2, p, engine=engine)
    _compare_presentations(g, o, synthdata.images(2, "fashion"), 350, synthdata.seeds(2, 1), 784, 6400, mode)
    assert o.stats()[1] > 0


@pytest.mark.parametrize("engine", ENGINES)
def test_C4_hf_variant(gpu, engine):
    p = O.params("hf", membrane_mode=1, init_seed=1)
    g, o = _pair(784, 6400, 2, p, engine=engine)
    _compare_presentations(g, o, synthdata.images(1, "fashion", start=5), 100, synthdata.seeds(1, 9), 784, 6400, 1)


@pytest.mark.parametrize("preset,wta,inh,stdp,lean", [("2b", 0, 0, 0, 1), ("8b", 0, 0, 0, 1), ("8b", 1, 0, 0, 1),
                                                      ("8b", 0, 1, 0, 0), ("8b", 0, 0, 1, 0)])
def test_lean_kernel_selection(gpu, preset, wta, inh, stdp, lean):
    """RESET inhibition with stochastic STDP (HARD or LAYER WTA) runs the lean kernel; HOLD inhibition, the
    deterministic arm, and SNN_ENGINE_EVENT_GENERAL run the general event kernel."""
    p = O.params(preset, wta_mode=wta, inh_mode=inh, stdp_mode=stdp)
    g, _ = _pair(784, 400, 8 if preset == "8b" else 2, p, engine=0)
    assert g.info()["lean"] == lean
    g2, _ = _pair(784, 400, 8 if preset == "8b" else 2, p, engine=2)
    assert g2.info()["lean"] == 0


# ------------------------------------------------------------------ C5: ensemble, one launch
@pytest.mark.parametrize("engine", ENGINES)
def test_C5_ensemble_present_many(gpu, engine):
    import paper_conf_date_shelm19_b200 as P
    nets, oracles, imgs, seeds = [], [], [], []
    for k in range(6):
        bits = (2, 4, 8)[k % 3]
        p = O.params({2: "2b", 4: "4b", 8: "8b"}[bits], membrane_mode=1, init_seed=1 + k, cluster_size=2)
        g, o = _pair(784, 400, bits, p, engine=engine)
        nets.append(g)
        oracles.append(o)
        imgs.append(synthdata.images(3, "mnist", start=10 * k))
        seeds.append(synthdata.seeds(3, base_seed=100 + k))
    P.present_many(nets, imgs, 120, seeds)
    for g, o, im, sd in zip(nets, oracles, imgs, seeds):
        for x, s in zip(im, sd):
            o.present(x, 120, int(s))
        assert np.array_equal(g.weights(), o.weights())
        assert np.array_equal(g.spikes(), o.spikes())


# ------------------------------------------------------------------ edge cases
@pytest.mark.parametrize("n_in,n_exc,bits", [(1, 1, 8), (33, 1, 2), (5, 65, 4), (784, 31, 2), (2000, 64, 8)])
@pytest.mark.parametrize("engine", ENGINES)
def test_ragged_shapes(gpu, engine, n_in, n_exc, bits):
    p = O.params("8b", membrane_mode=1, f_min_hz=20.0, f_max_hz=400.0, v_spike=30.0, init_seed=6)
    g, o = _pair(n_in, n_exc, bits, p, engine=engine)
    rng = np.random.default_rng(n_in * 7 + n_exc)
    imgs = rng.integers(0, 256, size=(2, n_in)).astype(np.uint8)
    _compare_presentations(g, o, imgs, 60, [3, 4], n_in, n_exc, 1)


@pytest.mark.parametrize("engine", ENGINES)
def test_zero_and_one_step(gpu, engine):
    p = O.params("8b", membrane_mode=1)
    g, o = _pair(784, 100, 8, p, engine=engine)
    img = synthdata.images(1)[0]
    for T in (0, 1, 2):
        g.present(img, T, 5)
        o.present(img, T, 5)
        assert np.array_equal(g.spikes(), o.spikes())
        assert np.array_equal(g.weights(), o.weights())
        _assert_state_equal(g, o, 784, 100, 1)


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("engine", ENGINES)
def test_stepwise_keep_state_and_reseed(gpu, engine, mode):
    """North-star protocol: after each single step (SNN_KEEP_STATE, t0 = t) the GPU state equals the
    oracle's; in fp32 mode v agrees to 1e-5 relative per step; the GPU can be reseeded from the
    oracle state at any point and continue identically."""
    import paper_conf_date_shelm19_b200 as P
    p = O.params("8b", membrane_mode=mode, init_seed=8)
    g, o = _pair(784, 64, 8, p, engine=engine)
    img = synthdata.images(1, "mnist", start=4)[0]
    for t in range(80):
        fl = O.ORACLE_KEEP_STATE if t else 0
        o.present_ex(img, 1, 21, flags=fl, t0=t)
        g.present_ex(img, 1, 21, flags=(P.SNN_KEEP_STATE if t else 0), t0=t)
        _assert_state_equal(g, o, 784, 64, mode)
        assert np.array_equal(g.weights(), o.weights())
        if t == 40:   # reseed the GPU from the oracle state
            g.set_state(o.state())
            g.set_weights(o.weights())


@pytest.mark.parametrize("engine", ENGINES)
def test_raster_input_ltp_ltd_paths(gpu, engine):
    """Encoder bypass (SNN_RASTER_INPUT) with forced post spikes: LTP / LTD counters and codes equal."""
    p = O.params("8b", i_ext=60.0, v_spike=1e-9, t_ref_steps=7, membrane_mode=1)
    g, o = _pair(784, 3, 8, p, engine=engine)
    rng = np.random.default_rng(3)
    raster = rng.integers(0, 2 ** 32, size=(40, 25), dtype=np.uint64).astype(np.uint32)
    raster &= rng.integers(0, 2 ** 32, size=(40, 25), dtype=np.uint64).astype(np.uint32)
    raster[:, -1] &= 0xFFFF
    g.present_raster(raster, 40, 99)
    o.present_raster(raster, 40, 99)
    assert np.array_equal(g.spikes(), o.spikes())
    assert np.array_equal(g.weights(), o.weights())
    assert np.array_equal(g.stats()[:6], o.stats()[:6])
    assert o.stats()[3] > 0 and o.stats()[5] > 0


# ------------------------------------------------------------------ event-engine rollback paths
@pytest.mark.parametrize("engine", ENGINES)
@pytest.mark.parametrize("mode,wta,stdp", [(0, 0, 0), (1, 0, 0), (1, 1, 0), (1, 1, 1)])
def test_inh_hold_mode(gpu, engine, mode, wta, stdp):
    """HOLD inhibition (inhibited neurons keep v): the event engine must re-simulate overrunning
    columns instead of the RESET shortcut."""
    p = O.params("8b", inh_mode=1, wta_mode=wta, stdp_mode=stdp, membrane_mode=mode, init_seed=12)
    g, o = _pair(784, 400, 8, p, engine=engine)
    _compare_presentations(g, o, synthdata.images(2, "mnist", start=40), 250, synthdata.seeds(2, 12), 784, 400, mode)
    assert o.stats()[1] > 0


@pytest.mark.parametrize("engine", ENGINES)
def test_undo_log_overflow_path(gpu, engine):
    """High input rates + gamma_dep = 1, tau_dep = 50: many LTD events per column-step overflow the
    per-thread undo log, exercising the partial-step undo and horizon epochs of the event engine."""
    p = O.params("2b", f_min_hz=200.0, f_max_hz=1000.0, gamma_dep=1.0, tau_dep=50.0, v_spike=0.5,
                 membrane_mode=1, init_seed=13)
    g, o = _pair(784, 256, 2, p, engine=engine)
    _compare_presentations(g, o, synthdata.images(2, "fashion", start=3), 120, synthdata.seeds(2, 13), 784, 256, 1)
    if engine in (0, 2):
        assert int(g.stats()[9]) > 0, "undo-log overflow path not exercised"


# ------------------------------------------------------------------ the exact benchmarked launch (bench.py)
def _batch_vs_oracle(p, n_in, n_exc, bits, imgs, T, seeds, engine=0, expect_lean=None):
    """One snn_present_batch launch of all images (weights resident in shared memory across the images,
    the in-launch image-boundary reset, window re-staging and per-image pre-drawn LTD reset) against the
    oracle presenting the same images one by one: per-image spike counts, final codes, the last image's
    raster, the state blob and the counters."""
    g, o = _pair(n_in, n_exc, bits, p, engine=engine)
    if expect_lean is not None:
        assert g.info()["lean"] == expect_lean
    counts = np.zeros(len(imgs), np.int32)
    g.reset_stats()
    g.present_batch(imgs, T, seeds, counts)
    oc, ost = [], np.zeros(6, np.int64)
    for img, sd in zip(imgs, seeds):
        o.present(img, T, int(sd))
        oc.append(int(O.unpack_bits(o.spikes(), n_exc).sum()))
        ost += o.stats()[:6].astype(np.int64)
    assert counts.tolist() == oc, "per-image post-spike counts"
    assert np.array_equal(g.weights(), o.weights()), "conductance codes after the batch"
    assert np.array_equal(g.spikes(), o.spikes()), "last image's output raster"
    assert np.array_equal(g.stats()[:6].astype(np.int64), ost), "counters summed over the batch"
    _assert_state_equal(g, o, n_in, n_exc, p["membrane_mode"])
    assert sum(oc) > 0
    return g


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("engine", [0, 2])
def test_C4_present_batch_vs_oracle(gpu, engine, mode):
    """bench.py's launch: 784 -> 6400, 2 bit, default cluster (16 CTAs; lean <2,2,*> kernel for engine 0),
    8 fashion images in ONE present_batch call."""
    p = O.params("2b", membrane_mode=mode, init_seed=1)
    g = _batch_vs_oracle(p, 784, 6400, 2, synthdata.images(8, "fashion", start=200), 350,
                         synthdata.seeds(8, base_seed=31), engine=engine, expect_lean=int(engine == 0))
    assert g.info()["cluster_size"] == 16


def test_C4_hf_present_batch_vs_oracle(gpu):
    """The 5-78 Hz "high frequency" row at T = 100, 8 images in one launch on the lean kernel."""
    p = O.params("hf", membrane_mode=1, init_seed=1)
    _batch_vs_oracle(p, 784, 6400, 2, synthdata.images(8, "fashion", start=300), 100,
                     synthdata.seeds(8, base_seed=37), expect_lean=1)


@pytest.mark.parametrize("n_exc,bits,preset,cs", [(400, 8, "8b", 0), (1600, 2, "2b", 0), (1600, 2, "2b", 2)])
def test_C2_C3_present_batch_vs_oracle(gpu, n_exc, bits, preset, cs):
    """Batches at the C2 / C3 shapes (other thread counts and cluster sizes than the bench's), 12 images per
    launch: the deferred column's tables cover 2 raw rows per thread, so their extent depends on the CTA size."""
    p = O.params(preset, membrane_mode=1, init_seed=3, cluster_size=cs)
    _batch_vs_oracle(p, 784, n_exc, bits, synthdata.images(12, "mnist", start=50), 350,
                     synthdata.seeds(12, base_seed=41), expect_lean=1)


def test_state_validation_matches_oracle(gpu):
    """Both sides reject a continuation that steps back in time and a state blob with timers at or after its
    t_next or negative countdowns, and accept the same valid blob."""
    import paper_conf_date_shelm19_b200 as P
    p = O.params("8b", membrane_mode=1)
    g, o = _pair(16, 4, 8, p)
    img = np.full(16, 200, np.uint8)
    g.present(img, 10, 3)
    o.present(img, 10, 3)
    with pytest.raises(P.SnnError) as e:
        g.present_ex(img, 5, 3, flags=P.SNN_KEEP_STATE, t0=9)
    assert e.value.rc == -1
    st = o.state()
    assert np.array_equal(g.state(), st)
    for bad_index, bad_value in ((4 + 4 + 0, -1), (4 + 8 + 1, int(st[2])), (4 + 12 + 3, int(st[2]) + 5)):
        b = st.copy()
        b[bad_index] = bad_value
        with pytest.raises(P.SnnError):
            g.set_state(b)
    g.set_state(st)


def test_floor_probe_and_profile_leave_learning_untouched(gpu):
    """bench.py's instruments: SNN_FLOOR_PROBE (the lean kernel's per-epoch synchronisation skeleton) changes no
    code, state or learning counter, and profiling (CUDA events around the presentation kernel) does not change
    results; the profile reports one kernel per presentation."""
    import paper_conf_date_shelm19_b200 as P
    p = O.params("2b", membrane_mode=1, init_seed=1)
    g, o = _pair(784, 512, 2, p)
    imgs, seeds = synthdata.images(6, "fashion", start=400), synthdata.seeds(6, base_seed=43)
    g.set_profile(True)
    g.present_batch(imgs[:3], 150, seeds[:3])
    ms, n = g.profile()
    assert n == 1 and ms > 0.0
    w0, st0, s0 = g.weights(), g.state(), g.stats()[:13].copy()
    counts = np.full(3, -1, np.int32)
    g.present_batch(imgs[3:], 150, seeds[3:], counts, flags=P.snn.SNN_FLOOR_PROBE)
    assert counts.tolist() == [0, 0, 0]
    assert np.array_equal(g.weights(), w0) and np.array_equal(g.state(), st0)
    assert np.array_equal(g.stats()[:13], s0)
    g.set_profile(False)
    for img, sd in zip(imgs[:3], seeds[:3]):
        o.present(img, 150, int(sd))
    assert np.array_equal(w0, o.weights())


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("start,base", [(400, 43), (0, 1), (123, 7), (777, 99), (2024, 5)])
def test_lean_short_tables_shared_thread(gpu, mode, start, base):
    """784 -> 512 at 2 bits on 16 CTAs of ONE warp: the deferred column's tables cover only ~5 steps (32 raw
    rows), so epochs end at table ends, re-simulations are frequent, and the deferred column often shares its
    thread with the next winner (regression: a later crossing reported by the deferred column's run ahead must
    not lend its key to an earlier crossing of the thread's other column)."""
    p = O.params("2b", membrane_mode=mode, init_seed=1)
    g, o = _pair(784, 512, 2, p)
    assert g.info()["threads"] == 32 and g.info()["lean"] == 1
    imgs, seeds = synthdata.images(4, "fashion", start=start), synthdata.seeds(4, base_seed=base)
    counts = np.zeros(4, np.int32)
    g.present_batch(imgs, 144, seeds, counts)
    oc = []
    for x, s in zip(imgs, seeds):
        o.present(x, 144, int(s))
        oc.append(int(O.unpack_bits(o.spikes(), 512).sum()))
    assert counts.tolist() == oc
    assert np.array_equal(g.weights(), o.weights())
    assert np.array_equal(g.spikes(), o.spikes())
    _assert_state_equal(g, o, 784, 512, mode)


def _fuzz_case(k):
    rng = np.random.default_rng(1000 + k)
    bits = int(rng.choice([2, 4, 8]))
    n_exc = int(rng.choice([33, 100, 256, 512, 1024]))
    fmin, fmax = [(1.0, 22.0), (5.0, 78.0), (10.0, 156.0)][int(rng.integers(3))]
    p = O.params({2: "2b", 4: "4b", 8: "8b"}[bits], membrane_mode=int(rng.integers(2)), init_seed=int(rng.integers(1, 99)),
                 wta_mode=int(rng.random() < 0.35),
                 f_min_hz=fmin, f_max_hz=fmax, t_ref_steps=int(rng.choice([1, 2, 5, 10])),
                 t_inh_steps=int(rng.choice([3, 5, 10])), v_spike=float(rng.choice([1.0, 2.0, 4.0])),
                 cluster_size=min(int(rng.choice([0, 0, 1, 2, 4])), (n_exc + 31) // 32))
    return p, bits, n_exc, int(rng.choice([60, 150, 350])), str(rng.choice(["mnist", "fashion"])), int(rng.integers(10000))


@pytest.mark.parametrize("k", range(48))
def test_lean_fuzz_vs_oracle(gpu, k):
    """Randomised configurations of the lean kernel's modes (RESET inhibition, stochastic STDP, HARD or LAYER
    WTA): widths, column counts, cluster sizes (one to many warps per CTA), input rates, refractory /
    inhibition lengths, current scale, membrane mode; 3 images per launch against the oracle presenting them
    one by one."""
    import paper_conf_date_shelm19_b200 as P
    p, bits, n_exc, T, kind, start = _fuzz_case(k)
    try:
        g, o = _pair(784, n_exc, bits, p)
    except P.SnnError as e:                       # a cluster size too small for the network's codes is refused
        assert e.rc == -5                         # (SNN_ESIZE); the library's own choice then runs the case
        p = dict(p, cluster_size=0)
        g, o = _pair(784, n_exc, bits, p)
    imgs, seeds = synthdata.images(3, kind, start=start), synthdata.seeds(3, base_seed=k + 1)
    counts = np.zeros(3, np.int32)
    g.present_batch(imgs, T, seeds, counts)
    oc = []
    for x, s in zip(imgs, seeds):
        o.present(x, T, int(s))
        oc.append(int(O.unpack_bits(o.spikes(), n_exc).sum()))
    assert counts.tolist() == oc
    assert np.array_equal(g.weights(), o.weights())
    assert np.array_equal(g.spikes(), o.spikes())
    _assert_state_equal(g, o, 784, n_exc, p["membrane_mode"])
