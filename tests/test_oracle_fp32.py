"""Pins of the oracle's 32-bit floating-point conductance arm (NEXT-2; R28) against what the
paper and mathematics fix, no GPU.

P:82 "stochastic STDP enables robust learning from 32-bit floating-point (accuracy 96.1%)";
P:89 §III-C "For 16-bit and 32-bit learning, after floating point calculation of change in conductance
dG, the result is rounded to a value that can be represented in the current bit width";
P:84 eqs.(4)(5) dG_p = alpha_p e^{-beta_p (G - G_min)/(G_max - G_min)}, dG_d = alpha_d e^{-beta_d (G_max - G)/(G_max - G_min)}.
None of the expected values comes from the CUDA path: they come from math.exp (libm), closed forms, or the
oracle's integer-code path on inputs where the two arms must agree exactly.
"""
import math

import numpy as np
import pytest

from oracle import oracle as O
import synthdata

from test_oracle_pins import _force_state, _spike_steps


def _p32(**kw):
    return O.params("16b", **kw)


def test_exp_recipe_matches_libm():
    """R28's binary64 e^y recipe against libm exp over the range eqs.(4)(5) use (y in [-beta, 0]) and beyond:
    relative error <= 2^-52 (2 ulp), exact at 0."""
    net = O.OracleNet(1, 1, 32, _p32())
    ys = np.concatenate([np.linspace(-40.0, 0.0, 20001), -np.random.default_rng(5).random(5000) * 3.0,
                         [-1e-300, -2.0 ** -60, -0.5 * math.log(2), 0.5 * math.log(2) - 1e-9, 1.0, 3.0]])
    worst = 0.0
    for y in ys:
        e = net.exp_recipe(float(y))
        ref = math.exp(float(y))
        worst = max(worst, abs(e - ref) / ref)
    assert worst <= 2.0 ** -52, worst
    assert net.exp_recipe(0.0) == 1.0
    for k in range(0, 30):              # reduction boundaries: y = -k ln2 (r = 0 up to the rounding of y)
        y = -k * math.log(2)
        assert abs(net.exp_recipe(y) - math.exp(y)) <= 2.0 ** -52 * math.exp(y)


@pytest.mark.parametrize("g_max", [1.0, 0.5])
def test_dg_is_eqs_4_5(g_max):
    """eqs.(4)(5) P:84 at G_min = 0: dG_p = alpha_p e^{-beta_p G/G_max}, dG_d = alpha_d e^{-beta_d (G_max - G)/G_max}.
    Distinct alpha/beta per branch and G_max != 1 so that a swapped parameter, a wrong sign or a dropped
    normalisation fails."""
    p = _p32(alpha_p=0.013, beta_p=2.5, alpha_d=0.0047, beta_d=3.5, g_max=g_max)
    net = O.OracleNet(1, 1, 32, p)
    for G in np.linspace(0.0, g_max, 41, dtype=np.float32):
        G = float(G)
        ep = 0.013 * math.exp(-2.5 * G / g_max)
        ed = 0.0047 * math.exp(-3.5 * (g_max - G) / g_max)
        assert abs(net.dg(False, G) - ep) <= 4e-16 * ep
        assert abs(net.dg(True, G) - ed) <= 4e-16 * ed
    # the endpoints: dG_p(G_min) = alpha_p, dG_d(G_max) = alpha_d
    assert net.dg(False, 0.0) == 0.013 and net.dg(True, g_max) == 0.0047


def test_validation():
    """R28: fp32 membranes and round-to-nearest only; set_weights takes G in [G_min, G_max]."""
    with pytest.raises(O.OracleError):
        O.OracleNet(4, 2, 32, _p32(membrane_mode=1))
    for rnd in (0, 2):
        with pytest.raises(O.OracleError):
            O.OracleNet(4, 2, 32, _p32(rounding=rnd))
    with pytest.raises(O.OracleError):
        O.OracleNet(4, 2, 12, _p32())
    net = O.OracleNet(4, 2, 32, _p32(g_max=0.75))
    assert net.weights().dtype == np.float32
    for bad in (0.76, -1e-6, float("nan"), float("inf")):
        w = np.full((4, 2), 0.5, np.float32)
        w[1, 1] = bad
        with pytest.raises(O.OracleError):
            net.set_weights(w)
    w = np.full((4, 2), 0.75, np.float32)
    net.set_weights(w)
    assert (net.weights() == w).all()


@pytest.mark.parametrize("g_max", [1.0, 0.75])
def test_init_uniform_grid(g_max):
    """R28 initial conductance: G = binary32(G_max (u >> 8) 2^-24): uniform on [0, G_max), mean G_max/2;
    at G_max = 1 exactly the 2^24-point grid."""
    net = O.OracleNet(784, 64, 32, _p32(g_max=g_max, init_seed=9))
    G = net.weights().astype(np.float64)
    assert G.min() >= 0.0 and G.max() < g_max
    if g_max == 1.0:
        k = G * 2.0 ** 24
        assert np.all(k == np.round(k))
    n = G.size
    assert abs(G.mean() - g_max / 2) <= 3 * g_max / math.sqrt(12 * n)
    # not the code-grid initialisation of the integer arms
    assert len(np.unique(G)) > n // 2


@pytest.mark.parametrize("v_spike,k_expected", [(3.0, 21), (5.0, 8), (10.0, 4)])
def test_integration_closed_form_first_spike(v_spike, k_expected):
    """eq.(3) I = v_pre sum_i g_i with binary32 g (R28): one input spiking every step (p = f dt = 1) with
    G = 1 gives the constant current I = v_spike; the first spike then follows the forward-Euler closed
    form of eq.(1) (the same table as the integer arms' i_ext pins: I = 3 -> 21, 5 -> 8, 10 -> 4 steps).
    A dropped v_spike or a stray LSB factor would move it."""
    p = _p32(v_spike=v_spike, f_min_hz=1000.0, f_max_hz=1000.0, gamma_pot=0.0, gamma_dep=0.0, t_ref_steps=0)
    net = O.OracleNet(1, 1, 32, p)
    net.set_weights(np.ones((1, 1), np.float32))
    net.present(np.full(1, 255, np.uint8), 60, seed=3)
    assert _spike_steps(net, 60)[0] + 1 == k_expected


def test_grid_weights_reduce_to_8bit_arm():
    """Special case: binary32 conductances on the 8-bit grid (G = q 2^-8) integrate exactly like the 8-bit
    arm (every partial sum is a multiple of 2^-8 below 2^10, exact in binary32, and S 2^-8 v_spike rounds
    once in both recipes), so with learning off both arms give identical rasters and membranes."""
    rng = np.random.default_rng(11)
    n_in, n_exc, T = 784, 40, 120
    q = rng.integers(0, 256, size=(n_in, n_exc)).astype(np.uint8)
    imgs = synthdata.images(3, "mnist", seed=20190325)
    for wta in (0, 1):
        kw = dict(gamma_pot=0.0, gamma_dep=0.0, wta_mode=wta, v_spike=2.5, f_min_hz=5.0, f_max_hz=78.0)
        a = O.OracleNet(n_in, n_exc, 8, _p32(**kw))
        b = O.OracleNet(n_in, n_exc, 32, _p32(**kw))
        a.set_weights(q)
        b.set_weights(q.astype(np.float32) / 256.0)
        spikes = 0
        for k in range(3):
            a.present(imgs[k], T, seed=100 + k)
            b.present(imgs[k], T, seed=100 + k)
            assert (a.spikes() == b.spikes()).all()
            assert (a.state() == b.state()).all()
            spikes += int(O.unpack_bits(a.spikes(), n_exc).sum())
        assert spikes > 5
        assert (b.weights() == q.astype(np.float32) / 256.0).all()


def _f32(x):
    return float(np.float32(x))


@pytest.mark.parametrize("t_ltp", [3, 20])
def test_det_arm_fp32_window_and_magnitudes(t_ltp):
    """Deterministic arm at 32 bits (R16 window, R28 magnitudes): at the post spike (t = P) every input of
    the winner moves by eq.(4) (fired within t_LTP steps, D = 0 included) or eq.(5) (fired earlier or never),
    G' = binary32(G +- dG) clamped to [0, G_max].  Expected values from libm exp."""
    P = t_ltp + 3
    steps = [P - t_ltp, P - t_ltp - 1, P, None]
    p = _p32(stdp_mode=1, t_ltp_steps=t_ltp, i_ext=60.0, v_spike=1e-9, t_ref_steps=100000)
    for G0 in (0.0, 0.3, 0.9996, 1.0, 0.002):
        G0 = _f32(G0)
        net = O.OracleNet(4, 1, 32, p)
        raster = np.zeros((P + 1, 1), np.uint32)
        for i, s in enumerate(steps):
            if s is not None:
                raster[s, 0] |= np.uint32(1 << i)
        net.set_weights(np.full((4, 1), G0, np.float32))
        _force_state(net, P)
        net.present_raster(raster, P + 1, seed=7, keep_state=True, t0=0)
        assert _spike_steps(net, P + 1) == [P]
        up = min(_f32(G0 + 0.01 * math.exp(-3.0 * G0)), 1.0)
        dn = max(_f32(G0 - 0.005 * math.exp(-3.0 * (1.0 - G0))), 0.0)
        want = [up, dn, up, dn]
        got = net.weights()[:, 0].astype(np.float64).tolist()
        assert got == want, (G0, got, want)
        st = net.stats()
        assert st[4] == 2 and st[5] == 2 and st[2] == 2 and st[3] == 2


def test_stoch_arm_fp32_ltp_certain_event():
    """Stochastic arm at 32 bits: the eqs.(6)(7) draw gates the event as at <= 8 bits and the event moves G
    by eq.(4) (R28).  gamma_pot = 1 at D = 0 makes P_pot = 1 (thr = 2^32): every input firing in the post
    step potentiates by exactly dG_p(G); inputs that never fired are untouched (no LTD without a post spike
    before them)."""
    n_in = 64
    p = _p32(i_ext=60.0, v_spike=1e-9, t_ref_steps=100000, gamma_pot=1.0, tau_pot=30.0, gamma_dep=0.0)
    net = O.OracleNet(n_in, 1, 32, p)
    G0 = np.linspace(0.0, 1.0, n_in, dtype=np.float32)
    net.set_weights(G0.reshape(n_in, 1))
    P = 4
    raster = np.zeros((P + 1, 2), np.uint32)
    raster[P, 0] = 0xFFFFFFFF                 # inputs 0..31 fire in the post step (D = 0)
    _force_state(net, P)
    net.present_raster(raster, P + 1, seed=5, keep_state=True, t0=0)
    assert _spike_steps(net, P + 1) == [P]
    got = net.weights()[:, 0]
    for i in range(n_in):
        g = float(G0[i])
        want = min(_f32(g + 0.01 * math.exp(-3.0 * g)), 1.0) if i < 32 else g
        assert float(got[i]) == want, (i, float(got[i]), want)
    st = net.stats()
    assert st[4] == 32 and st[5] == 32


def test_stoch_arm_fp32_ltd_magnitude_and_clamp():
    """LTD at 32 bits: a pre spike D steps after the post spike depresses with probability P_dep(D) (eq.(7),
    gating as at <= 8 bits) and by eq.(5) when it does (R28), clamped at G_min = 0.  tau_dep large makes
    P_dep(3) = e^{-0.02} ~ 0.98; each event is checked against the magnitude, each non-event against no change."""
    n_in = 96
    p = _p32(i_ext=60.0, v_spike=1e-9, t_ref_steps=100000, gamma_pot=0.0, gamma_dep=1.0, tau_dep=150.0)
    net = O.OracleNet(n_in, 1, 32, p)
    G0 = np.concatenate([np.linspace(0.0, 1.0, n_in - 8, dtype=np.float32), np.full(8, 1e-4, np.float32)])
    net.set_weights(G0.reshape(n_in, 1))
    P = 2
    T = P + 4
    wi = (n_in + 31) // 32
    raster = np.zeros((T, wi), np.uint32)
    raster[P + 3, :] = 0xFFFFFFFF             # all inputs fire 3 steps after the post spike
    _force_state(net, P)
    net.present_raster(raster, T, seed=5, keep_state=True, t0=0)
    assert _spike_steps(net, T)[0] == P
    got = net.weights()[:, 0]
    moved = 0
    for i in range(n_in):
        g = float(G0[i])
        dn = max(_f32(g - 0.005 * math.exp(-3.0 * (1.0 - g))), 0.0)
        assert float(got[i]) in (g, dn)
        moved += float(got[i]) != g
    assert (got[-8:] == 0.0).sum() >= 5            # 1e-4 - dG_d(1e-4) < 0 clamps to G_min
    st = net.stats()
    assert st[2] == n_in and st[3] >= n_in - 8 and moved >= n_in - 9
