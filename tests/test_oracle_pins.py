"""Pins of the CPU oracle against what the paper and mathematics fix (no GPU).

Each test names the passage of /root/reference/PAPER.md (P:<line>) or the DESIGN.md reading
it pins.  None of the expected values comes from the CUDA path.
"""
import math

import numpy as np
import pytest

from oracle import oracle as O
import synthdata

MODES = [0, 1]  # membrane_mode: 0 fp32 recipe, 1 Q15.16 fixed recipe


# ------------------------------------------------------------------ Philox4x32-10 (R13)
def test_philox_known_answers():
    # Random123 known-answer vectors for philox4x32_10 (Salmon et al. SC'11 reference code).
    assert O.philox4x32_10([0, 0, 0, 0], [0, 0]) == [0x6627E8D5, 0xE169C58D, 0xBC57AC4C, 0x9B00DBD8]
    assert O.philox4x32_10([0xFFFFFFFF] * 4, [0xFFFFFFFF] * 2) == [0x408F276D, 0x41C83B0E, 0xA20BC7C6, 0x6D5451FD]
    assert O.philox4x32_10([0x243F6A88, 0x85A308D3, 0x13198A2E, 0x03707344], [0xA4093822, 0x299F31D0]) == \
        [0xD16CFE09, 0x94FDCCEB, 0x5001E420, 0x24126EA1]


# ------------------------------------------------------------------ LIF closed form, eqs.(1)(2)
def _closed_form_first_spike(I, v0, p=O.BASE):
    """Forward Euler (R1, R2) under constant I: v_k = v_inf + (v0 - v_inf) lam^k, lam = 1 + b dt;
    first k with v_k > V_th (strict, eq.(2))."""
    a, b, c, vth, dt = p["a"], p["b"], p["c"], p["v_th"], p["dt_ms"]
    lam = 1.0 + b * dt
    vinf = -(a + c * I) / b
    if vinf <= vth:
        return None, None
    x = math.log((vinf - vth) / (vinf - v0)) / math.log(lam)
    return math.floor(x) + 1, x - math.floor(x)


def _spike_steps(net, T):
    r = O.unpack_bits(net.spikes(), net.n_exc)
    return [int(t) for t in np.nonzero(r[:, 0])[0]]


# Values restated in SURVEY §8(c) pins table: from v0 = -70: I=2.6 -> 83, 2.7 -> 34, 3 -> 21, 4 -> 12,
# 5 -> 8, 10 -> 4, 20 -> 2 steps; rheobase I_rh = -(a + b V_th)/c = 2.59943.
FIRST_SPIKE = {2.6: 83, 2.7: 34, 3.0: 21, 4.0: 12, 5.0: 8, 10.0: 4, 20.0: 2}


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("I,k_expected", sorted(FIRST_SPIKE.items()))
def test_lif_first_spike_closed_form(mode, I, k_expected):
    k, frac = _closed_form_first_spike(I, -70.0)
    assert k == k_expected and 1e-3 < frac < 1 - 1e-3
    p = O.params("8b", i_ext=I, f_min_hz=0.0, f_max_hz=0.0, gamma_pot=0.0, gamma_dep=0.0,
                 membrane_mode=mode, t_ref_steps=0)
    net = O.OracleNet(1, 1, 8, p)
    net.present(np.zeros(1, np.uint8), 200, seed=7)
    steps = _spike_steps(net, 200)
    assert steps[0] + 1 == k_expected   # step index t performs Euler step k = t + 1


def test_rheobase():
    p = O.BASE
    i_rh = -(p["a"] + p["b"] * p["v_th"]) / p["c"]
    assert abs(i_rh - 2.59943) < 1e-5
    for mode in MODES:
        below = O.params("8b", i_ext=2.59, f_min_hz=0.0, f_max_hz=0.0, gamma_pot=0.0, gamma_dep=0.0,
                         membrane_mode=mode)
        net = O.OracleNet(1, 1, 8, below)
        net.present(np.zeros(1, np.uint8), 1000, seed=1)
        assert _spike_steps(net, 1000) == []


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("I,t_ref", [(3.0, 0), (5.0, 0), (3.0, 5), (10.0, 3)])
def test_lif_interspike_interval(mode, I, t_ref):
    """Fig. 1(a) f-I curve: ISI = t_ref + k(I, from v_reset); I=3 -> 25 steps (40 Hz), I=5 -> 11."""
    k_reset, frac = _closed_form_first_spike(I, -74.7)
    assert 1e-3 < frac < 1 - 1e-3
    if t_ref == 0:
        assert k_reset == {3.0: 25, 5.0: 11}[I]
    p = O.params("8b", i_ext=I, f_min_hz=0.0, f_max_hz=0.0, gamma_pot=0.0, gamma_dep=0.0,
                 membrane_mode=mode, t_ref_steps=t_ref)
    net = O.OracleNet(1, 1, 8, p)
    net.present(np.zeros(1, np.uint8), 300, seed=3)
    steps = _spike_steps(net, 300)
    assert len(steps) >= 3
    assert all(b - a == t_ref + k_reset for a, b in zip(steps, steps[1:]))


def test_lif_fp32_recipe_tracks_exact_euler():
    """fp32 recipe (R12) vs the exact Euler update in double: per-step relative error < 1e-6
    (north_star tolerance is 1e-5 relative per step)."""
    p = O.params("8b")
    net = O.OracleNet(1, 1, 8, p)
    rng = np.random.default_rng(0)
    lsb = 2.0 ** -8
    for _ in range(2000):
        v = float(np.float32(rng.uniform(-80, -55)))
        S = int(rng.integers(0, 2560))            # I = v_spike * LSB * S in [0, 20]
        I = p["v_spike"] * lsb * S
        exact = v + p["dt_ms"] * (p["a"] + p["b"] * v + p["c"] * I)
        got = net.lif_step_fp32(v, S)
        assert abs(got - exact) <= 1e-6 * abs(exact)


def test_lif_fixed_recipe_tracks_exact_euler():
    """Q15.16 recipe (R12): one step within 4 LSB (2^-16 mV) + constant-quantisation error of exact Euler."""
    p = O.params("8b")
    net = O.OracleNet(1, 1, 8, p)
    rng = np.random.default_rng(1)
    lsb = 2.0 ** -8
    for _ in range(2000):
        vq = int(rng.integers(-80 << 16, -55 << 16))
        v = vq / 65536.0
        S = int(rng.integers(0, 2560))
        I = p["v_spike"] * lsb * S
        exact = v + p["dt_ms"] * (p["a"] + p["b"] * v + p["c"] * I)
        got = net.lif_step_fixed(vq, S) / 65536.0
        assert abs(got - exact) <= 4.0 / 65536.0 + S * 2.0 ** -32 * 2


# ------------------------------------------------------------------ integration, eq.(3), with saturating input
@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("qval,k_expected", [(1, 20), (2, 7)])
def test_saturating_input_integration(mode, qval, k_expected):
    """f_min = f_max = 1000 Hz -> p = 1: all 784 inputs spike every step, I = v_spike * LSB * sum q.
    8 bit, v_spike = 1: q=1 -> I = 784/256 = 3.0625 -> first spike k=20; q=2 -> I=6.125 -> k=7."""
    p = O.params("8b", v_spike=1.0, f_min_hz=1000.0, f_max_hz=1000.0, gamma_pot=0.0, gamma_dep=0.0,
                 membrane_mode=mode)
    net = O.OracleNet(784, 3, 8, p)
    net.set_weights(np.full((784, 3), qval, np.uint8))
    net.present(np.full(784, 17, np.uint8), 40, seed=11)
    assert O.unpack_bits(net.input_raster(), 784).all()
    k, _ = _closed_form_first_spike(784 * qval / 256.0, -70.0)
    assert k == k_expected
    r = O.unpack_bits(net.spikes(), 3)
    first = np.nonzero(r.any(axis=1))[0][0]
    assert first + 1 == k_expected
    assert r[first].tolist() == [True, False, False]       # identical columns: tie -> lowest index (R7)


# ------------------------------------------------------------------ encoder, §III-B + R8
def test_encoder_threshold_value():
    net = O.OracleNet(1, 1, 8, O.params("8b"))
    thr = net.lut(0)
    assert int(thr[255]) == 94489280          # floor(0.022 * 2^32), 22 Hz at dt = 1 ms
    assert int(thr[0]) == 4294967             # floor(0.001 * 2^32), 1 Hz


@pytest.mark.parametrize("fmin,fmax,x", [(1.0, 22.0, 255), (1.0, 22.0, 0), (1.0, 22.0, 128),
                                         (5.0, 78.0, 255), (5.0, 78.0, 60)])
def test_encoder_rate_within_3_sigma(fmin, fmax, x):
    """Empirical spike count within 3 sigma of Binomial(N, f dt), f = f_min + (f_max - f_min) x / 255."""
    T, n = 1000, 784
    p = O.params("8b", f_min_hz=fmin, f_max_hz=fmax, gamma_pot=0.0, gamma_dep=0.0)
    net = O.OracleNet(n, 1, 8, p)
    net.present(np.full(n, x, np.uint8), T, seed=12345)
    count = int(O.unpack_bits(net.input_raster(), n).sum())
    prob = (fmin + (fmax - fmin) * x / 255.0) * 1e-3
    N = T * n
    assert abs(count - N * prob) <= 3.0 * math.sqrt(N * prob * (1 - prob))
    assert net.stats()[0] == count


def test_encoder_rate_proportional_to_intensity():
    """'For darker pixels, the spiking frequency is higher': per-pixel rates over a 0..255 ramp."""
    T, n = 4000, 256
    p = O.params("8b", gamma_pot=0.0, gamma_dep=0.0, f_min_hz=5.0, f_max_hz=78.0)
    net = O.OracleNet(n, 1, 8, p)
    img = np.arange(256, dtype=np.uint8)
    net.present(img, T, seed=99)
    counts = O.unpack_bits(net.input_raster(), n).sum(axis=0)
    prob = (5.0 + 73.0 * img / 255.0) * 1e-3
    z = (counts - T * prob) / np.sqrt(T * prob * (1 - prob))
    assert np.abs(z).max() < 4.5
    slope = np.polyfit(img.astype(float), counts / T, 1)[0]
    assert abs(slope - 73e-3 / 255.0) < 0.1 * 73e-3 / 255.0


# ------------------------------------------------------------------ stochastic STDP probabilities, eqs.(6)(7)
def _force_state(net, cnt0):
    st = net.state()
    n_exc, n_in = net.n_exc, net.n_in
    v = np.full(n_exc, net.p["v_init"], np.float32).view(np.int32)
    st[4:4 + n_exc] = v
    st[4 + n_exc:4 + 2 * n_exc] = cnt0
    st[4 + 2 * n_exc:4 + 3 * n_exc] = -1
    st[4 + 3 * n_exc:4 + 3 * n_exc + n_in] = -1
    st[2] = 0
    net.set_state(st)


@pytest.mark.parametrize("D", [0, 7, 30, 90])
def test_ltp_probability_matches_eq6(D):
    """Pre spike at t=0, post spike forced at t=D (held D steps, then i_ext >> rheobase):
    P(q -> q+1) = gamma_pot exp(-D / tau_pot), Dt = t_post - t_pre = D >= 0 (R10)."""
    n_in, reps = 784, 100
    p = O.params("8b", i_ext=60.0, v_spike=1e-9, t_ref_steps=100000, gamma_dep=0.0)
    net = O.OracleNet(n_in, 1, 8, p)
    wi = (n_in + 31) // 32
    raster = np.zeros((D + 1, wi), np.uint32)
    raster[0, :] = 0xFFFFFFFF
    raster[0, -1] = (1 << (n_in % 32)) - 1 if n_in % 32 else 0xFFFFFFFF
    up = 0
    for r in range(reps):
        net.set_weights(np.zeros((n_in, 1), np.uint8))
        _force_state(net, D)
        net.present_raster(raster, D + 1, seed=1000 + r, keep_state=True, t0=0)
        assert _spike_steps(net, D + 1) == [D]
        w = net.weights()
        assert set(np.unique(w).tolist()) <= {0, 1}
        up += int(w.sum())
    N = n_in * reps
    P = 0.5 * math.exp(-D / 30.0)
    assert abs(up - N * P) <= 3.0 * math.sqrt(N * P * (1 - P))


@pytest.mark.parametrize("D", [1, 5, 20])
def test_ltd_probability_matches_eq7(D):
    """Post spike at t=0, pre spikes at t=D: P(q -> q-1) = gamma_dep exp(Dt / tau_dep), Dt = -D (R10)."""
    n_in, reps = 784, 100
    p = O.params("8b", i_ext=60.0, v_spike=1e-9, t_ref_steps=100000, gamma_pot=0.0)
    net = O.OracleNet(n_in, 1, 8, p)
    wi = (n_in + 31) // 32
    raster = np.zeros((D + 1, wi), np.uint32)
    raster[D, :] = 0xFFFFFFFF
    raster[D, -1] = (1 << (n_in % 32)) - 1 if n_in % 32 else 0xFFFFFFFF
    down = 0
    for r in range(reps):
        net.set_weights(np.ones((n_in, 1), np.uint8))
        _force_state(net, 0)
        net.present_raster(raster, D + 1, seed=5000 + r, keep_state=True, t0=0)
        assert _spike_steps(net, D + 1) == [0]
        down += int((net.weights() == 0).sum())
    N = n_in * reps
    P = 0.5 * math.exp(-D / 10.0)
    assert abs(down - N * P) <= 3.0 * math.sqrt(N * P * (1 - P))


def test_lut_horizons():
    """Table I taus: horizon where gamma e^{-D/tau} 2^32 drops below 1."""
    def L(preset, which):
        return len(O.OracleNet(1, 1, 8, O.params(preset)).lut(which))
    for preset, which, tau, gamma in [("2b", 1, 20.0, 0.2), ("hf", 1, 80.0, 0.3), ("hf", 2, 5.0, 0.2),
                                      ("8b", 1, 30.0, 0.5), ("2b", 2, 10.0, 0.2)]:
        expect = math.floor(tau * math.log(gamma * 2 ** 32)) + 1
        assert L(preset, which) == expect
    # last D with a nonzero threshold, tau=20 / gamma=0.2: floor(20 ln(0.2 2^32)) = 411
    assert L("2b", 1) - 1 == 411


# ------------------------------------------------------------------ quantisation / WTA invariants
def _stepwise_run(p, n_in, n_exc, bits, img, T, seed):
    net = O.OracleNet(n_in, n_exc, bits, p)
    ws, rs, sts = [net.weights()], [], []
    for t in range(T):
        net.present_ex(img, 1, seed, flags=(O.ORACLE_KEEP_STATE if t else 0), t0=t)
        ws.append(net.weights())
        rs.append(O.unpack_bits(net.spikes(), n_exc)[0])
        sts.append(O.unpack_state(net.state(), n_in, n_exc))
    return net, ws, np.array(rs), sts


@pytest.mark.parametrize("bits,preset", [(8, "8b"), (2, "2b"), (4, "4b")])
def test_invariants_stepwise(bits, preset):
    n_in, n_exc, T = 784, 24, 120
    p = O.params(preset)
    img = synthdata.images(1, "mnist")[0]
    net, ws, raster, sts = _stepwise_run(p, n_in, n_exc, bits, img, T, seed=77)
    qmax = 2 ** bits - 1
    for w0, w1 in zip(ws, ws[1:]):
        assert w1.max() <= qmax
        d = w1.astype(int) - w0.astype(int)
        assert set(np.unique(d).tolist()) <= {-1, 0, 1}         # one LSB per synapse per step
    assert raster.sum(axis=1).max() <= 1                         # HARD WTA: <= 1 spike per step (R7)
    spikes = [(t, int(np.nonzero(raster[t])[0][0])) for t in range(T) if raster[t].any()]
    assert len(spikes) >= 2, "test net must spike"
    t_first = spikes[0][0]
    for t in range(t_first):                                    # no STDP before the first post spike
        assert np.array_equal(ws[t + 1], ws[0])
    for (t, j), nxt in zip(spikes, spikes[1:]):
        gap = nxt[0] - t
        assert gap > (p["t_ref_steps"] if nxt[1] == j else p["t_inh_steps"])
    for t, j in spikes:                                          # spike timer updated
        assert sts[t]["last_post"][j] == t

    # the same T steps in one presentation give identical results (t0 / state plumbing)
    one = O.OracleNet(n_in, n_exc, bits, p)
    one.present(img, T, seed=77)
    assert np.array_equal(one.weights(), ws[-1])
    assert np.array_equal(O.unpack_bits(one.spikes(), n_exc), raster)


def test_gamma_zero_freezes_weights():
    p = O.params("8b", gamma_pot=0.0, gamma_dep=0.0)
    net = O.OracleNet(784, 16, 8, p)
    w0 = net.weights()
    for k, img in enumerate(synthdata.images(3, "fashion")):
        net.present(img, 150, seed=k)
    assert np.array_equal(net.weights(), w0)
    assert net.stats()[1] > 0


def test_initial_weights_uniform_on_grid():
    """R4 (P:90 truncated): codes uniform on {0..q_max}; chi-square over the grid."""
    for bits in (2, 4, 8):
        net = O.OracleNet(784, 400, bits, O.params("8b", init_seed=3))
        w = net.weights().reshape(-1)
        k = 2 ** bits
        counts = np.bincount(w, minlength=k)
        assert counts.size == k
        e = w.size / k
        chi2 = ((counts - e) ** 2 / e).sum()
        assert chi2 < k - 1 + 5 * math.sqrt(2 * (k - 1))


def test_tie_resolves_to_lowest_index_hard_and_all_spike_layer():
    n_in = 784
    img = np.full(n_in, 200, np.uint8)
    w = np.full((n_in, 4), 40, np.uint8)
    for wta, expect_first in [(0, [True, False, False, False]), (1, [True, True, True, True])]:
        p = O.params("8b", wta_mode=wta, gamma_pot=0.0, gamma_dep=0.0)
        net = O.OracleNet(n_in, 4, 8, p)
        net.set_weights(w)
        net.present(img, 60, seed=5)
        r = O.unpack_bits(net.spikes(), 4)
        first = np.nonzero(r.any(axis=1))[0][0]
        assert r[first].tolist() == expect_first
        st = O.unpack_state(net.state(), n_in, 4)
        if wta == 1:   # >= 2 spikers: everyone inhibited for t_inh (R7), incl. the spikers
            assert r[first + 1: first + 1 + 10].sum() == 0


def test_layer_single_spiker_not_self_inhibited():
    """LAYER mode (R7): a lone spiker keeps t_ref (not t_inh); the others get t_inh."""
    n_in = 64
    p = O.params("8b", wta_mode=1, gamma_pot=0.0, gamma_dep=0.0, t_ref_steps=2, t_inh_steps=7,
                 f_min_hz=1000.0, f_max_hz=1000.0, v_spike=1.0)
    net = O.OracleNet(n_in, 2, 8, p)
    w = np.zeros((n_in, 2), np.uint8)
    w[:, 0] = 255
    net.set_weights(w)
    net.present(np.zeros(n_in, np.uint8), 12, seed=1)
    r = O.unpack_bits(net.spikes(), 2)
    t0 = int(np.nonzero(r[:, 0])[0][0])
    st_cnt = None
    # the lone spiker re-fires after t_ref + (steps to threshold), well before t_inh would allow
    t1 = int(np.nonzero(r[t0 + 1:, 0])[0][0]) + t0 + 1
    assert t1 - t0 <= 2 + 2
    assert not r[:, 1].any()


# ------------------------------------------------------------------ deterministic arm, eqs.(4)(5)(8), R16/R17
def _det_run(bits, rounding, q_init, pre_fires, reps=1, seed0=0):
    """One post spike at t=5 (held 5 steps); inputs in `pre_fires` spike at t=2 (inside the window)."""
    n_in = len(pre_fires)
    p = O.params("16b", stdp_mode=1, rounding=rounding, i_ext=60.0, v_spike=1e-9, t_ref_steps=100000)
    net = O.OracleNet(n_in, 1, bits, p)
    wi = (n_in + 31) // 32
    raster = np.zeros((6, wi), np.uint32)
    for i, f in enumerate(pre_fires):
        if f:
            raster[2, i // 32] |= np.uint32(1 << (i % 32))
    outs = []
    for r in range(reps):
        net.set_weights(np.full((n_in, 1), q_init, net.code_dtype))
        _force_state(net, 5)
        net.present_raster(raster, 6, seed=seed0 + r, keep_state=True, t0=0)
        assert _spike_steps(net, 6) == [5]
        outs.append(net.weights()[:, 0].astype(int))
    return np.array(outs)


def test_det_arm_hand_values_8bit():
    """eq.(4) at G = 0, 8 bit: dG_p = alpha_p e^0 = 0.01 = 2.56 LSB -> trunc 2, nearest 3.
    eq.(5) at G = 255/256: dG_d = 0.005 e^{-3/256} = 1.2651 LSB -> trunc 1, nearest 1.
    eq.(5) at G = 128/256: 0.005 e^{-1.5} = 0.2856 LSB -> trunc 0, nearest 0."""
    fires = [True, False]
    assert _det_run(8, 0, 0, fires)[0].tolist() == [2, 0]
    assert _det_run(8, 1, 0, fires)[0].tolist() == [3, 0]
    assert _det_run(8, 0, 255, fires)[0].tolist() == [255, 254]   # pot saturates at q_max, dep by 1
    assert _det_run(8, 1, 255, fires)[0].tolist() == [255, 254]
    assert _det_run(8, 1, 128, fires)[0].tolist() == [128 + 1, 128]  # 2.56 e^{-1.5} = 0.571 -> 1; dep 0


@pytest.mark.parametrize("t_ltp", [0, 3, 20])
def test_det_arm_ltp_window_boundary(t_ltp):
    """R16 window (eqs.(4)(5), Querlioz-style rule): at the post spike of W (t = P), input i takes
    eq.(4) iff it fired and P - last_pre_i <= t_LTP, else eq.(5).  Four inputs per code value fire exactly
    t_LTP steps before the post spike (inside: LTP), t_LTP + 1 before (outside: LTD), in the post step itself
    (D = 0: LTP), and never (LTD).  8 bit, nearest: q = 128 -> LTP 2.56 e^{-1.5} = 0.571 -> +1, LTD 0.286 -> 0;
    q = 240 -> LTP 2.56 e^{-2.8125} = 0.154 -> 0, LTD 1.28 e^{-0.1875} = 1.061 -> -1."""
    P = t_ltp + 3
    steps = [P - t_ltp, P - t_ltp - 1, P, None]
    p = O.params("16b", stdp_mode=1, rounding=1, t_ltp_steps=t_ltp, i_ext=60.0, v_spike=1e-9,
                 t_ref_steps=100000)
    expect = {128: [129, 128, 129, 128], 240: [240, 239, 240, 239]}
    for q0, want in expect.items():
        net = O.OracleNet(4, 1, 8, p)
        raster = np.zeros((P + 1, 1), np.uint32)
        for i, s in enumerate(steps):
            if s is not None:
                raster[s, 0] |= np.uint32(1 << i)
        net.set_weights(np.full((4, 1), q0, np.uint8))
        _force_state(net, P)
        net.present_raster(raster, P + 1, seed=7, keep_state=True, t0=0)
        assert _spike_steps(net, P + 1) == [P]
        assert net.weights()[:, 0].astype(int).tolist() == want, (q0, t_ltp)


def test_det_arm_2bit_truncation_never_learns():
    """Q0.2: dG_p <= 0.01 = 0.04 LSB, dG_d <= 0.005 = 0.02 LSB -> truncation and nearest give 0:
    consistent with Table II Q0.2 baseline ~ chance (9.6 %)."""
    for rnd in (0, 1):
        out = _det_run(2, rnd, 1, [True, False, True, False])
        assert out[0].tolist() == [1, 1, 1, 1]


def test_det_arm_stochastic_rounding_eq8():
    """eq.(8): P_round_up = frac(dG / LSB).  8 bit, q=0: 2.56 -> 3 w.p. 0.56, else 2."""
    out = _det_run(8, 2, 0, [True] * 64, reps=60)
    vals = out.reshape(-1)
    assert set(np.unique(vals).tolist()) <= {2, 3}
    N = vals.size
    k = int((vals == 3).sum())
    assert abs(k - 0.56 * N) <= 3 * math.sqrt(N * 0.56 * 0.44)


def test_det_arm_hand_values_16bit():
    """16 bit (frac 16, LSB 2^-16): eq.(4) at G = 0: 0.01 * 65536 = 655.36 LSB -> trunc 655, nearest 655;
    eq.(5) at G = 65535/65536: 0.005 e^{-3/65536} * 65536 = 327.665 LSB -> trunc 327, nearest 328."""
    fires = [True, False]
    assert _det_run(16, 0, 0, fires)[0].tolist() == [655, 0]
    assert _det_run(16, 1, 0, fires)[0].tolist() == [655, 0]
    assert _det_run(16, 0, 65535, fires)[0].tolist() == [65535, 65535 - 327]
    assert _det_run(16, 1, 65535, fires)[0].tolist() == [65535, 65535 - 328]


def _stoch16_run(rounding, q_init, pre_step, reps, gamma_dep=0.0, tau_dep=10.0):
    """16-bit stochastic arm (R27): one post spike forced at t=5; 64 inputs spike at `pre_step`
    (5 -> LTP with D = 0, 6 -> LTD with D = 1)."""
    n_in = 64
    p = O.params("16b", rounding=rounding, gamma_pot=1.0, gamma_dep=gamma_dep, tau_dep=tau_dep, i_ext=60.0,
                 v_spike=1e-9, t_ref_steps=100000)
    net = O.OracleNet(n_in, 1, 16, p)
    raster = np.zeros((8, 2), np.uint32)
    raster[pre_step, :] = 0xFFFFFFFF
    outs = []
    for r in range(reps):
        net.set_weights(np.full((n_in, 1), q_init, np.uint16))
        _force_state(net, 5)
        net.present_raster(raster, 8, seed=100 + r, keep_state=True, t0=0)
        assert _spike_steps(net, 8) == [5]
        outs.append(net.weights()[:, 0].astype(int))
    return np.concatenate(outs)


def test_stochastic_arm_16bit_magnitudes():
    """P:89 "For 16-bit ... after floating point calculation of change in conductance dG, the result is
    rounded": an LTP event moves q by eq.(4) rounded (trunc / nearest: 655), and with eq.(8) by 655 or 656
    with P(656) = 0.36; gamma_pot = 1 at D = 0 makes the event certain (eq.(6))."""
    assert set(_stoch16_run(0, 0, 5, 2).tolist()) == {655}
    assert set(_stoch16_run(1, 0, 5, 2).tolist()) == {655}
    v = _stoch16_run(2, 0, 5, 40)
    assert set(v.tolist()) <= {655, 656}
    N, k = v.size, int((v == 656).sum())
    assert abs(k - 0.36 * N) <= 3 * math.sqrt(N * 0.36 * 0.64)


def test_stochastic_arm_16bit_ltd():
    """A pre spike one step after the post spike: LTD event w.p. P_dep(1) = gamma_dep e^{-1/tau_dep}
    (eq.(7)), moving q_max by eq.(5) rounded to nearest (328 LSB)."""
    v = _stoch16_run(1, 65535, 6, 40, gamma_dep=1.0, tau_dep=100.0)
    assert set(v.tolist()) <= {65535, 65535 - 328}
    N, k = v.size, int((v == 65535 - 328).sum())
    P = math.exp(-1.0 / 100.0)
    assert abs(k - P * N) <= 3 * math.sqrt(N * P * (1 - P)) + 1


# ------------------------------------------------------------------ validation
@pytest.mark.parametrize("bad", [dict(gamma_pot=1.5), dict(tau_dep=0.0), dict(f_max_hz=2000.0),
                                 dict(f_min_hz=30.0, f_max_hz=20.0), dict(wta_mode=3), dict(g_min=0.1),
                                 dict(rounding=7), dict(tau_pot=1e6)])
def test_invalid_params_rejected(bad):
    with pytest.raises(O.OracleError) as e:
        O.OracleNet(784, 10, 8, O.params("8b", **bad))
    assert e.value.rc == -1


@pytest.mark.parametrize("bits", [0, 1, 3, 12, 24, 64])
def test_invalid_bits_rejected(bits):
    with pytest.raises(O.OracleError):
        O.OracleNet(784, 10, bits, O.params("8b"))


def test_state_validation_rejects_timers_from_the_future():
    """Input validation: a continued presentation may not start before the stored state's next
    step, and a state blob whose spike timers are not before its t_next (or whose countdowns are negative)
    is rejected, so Dt = t - last >= 1 always indexes the eqs.(6)(7) tables."""
    p = O.params("8b")
    net = O.OracleNet(16, 4, 8, p)
    net.present(np.full(16, 200, np.uint8), 10, seed=3)
    with pytest.raises(O.OracleError):
        net.present_ex(np.full(16, 200, np.uint8), 5, 3, flags=O.ORACLE_KEEP_STATE, t0=9)
    net.present_ex(np.full(16, 200, np.uint8), 5, 3, flags=O.ORACLE_KEEP_STATE, t0=10)   # t0 == t_next is fine
    st = net.state()
    for bad_index, bad_value in ((4 + 4 + 0, -1), (4 + 8 + 1, int(st[2])), (4 + 12 + 3, int(st[2]) + 5)):
        b = st.copy()
        b[bad_index] = bad_value
        with pytest.raises(O.OracleError):
            net.set_state(b)
    net.set_state(st)
