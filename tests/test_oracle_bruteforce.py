"""Brute-force pin of the whole per-step loop (SURVEY §8(c) "Whole step" row).

A 4-input / 2-neuron network in Q15.16 fixed-point mode is enumerated EXACTLY: every input
spike pattern (Bernoulli p_i = f_i dt) and every stochastic-STDP branch (eqs.(6)(7),
P:85) with its real-valued probability, giving the exact distribution of (final codes,
output raster).  The oracle's Monte-Carlo over 10^5 seeds must match it (chi-square).  The
enumerator is a third, independent statement of the step (no Philox, no threshold tables),
so it pins the phase order (encode -> integrate -> LIF -> WTA -> LTD -> LTP -> timers, R14),
the Dt offsets and signs (R10), the clamps and the WTA/inhibition rules (R7).
"""
import itertools
import math
from collections import defaultdict

import numpy as np
import pytest
from scipy import stats as sst

from oracle import oracle as O

N_IN, N_EXC, BITS, T = 4, 2, 2, 3
IMAGE = np.array([255, 200, 120, 40], np.uint8)
Q0 = np.array([[1, 3], [2, 0], [3, 1], [0, 2]], np.uint8)

PARAMS = O.params(
    "2b", membrane_mode=1, v_init=-61.0, v_spike=12.0, t_ref_steps=1, t_inh_steps=2,
    f_min_hz=50.0, f_max_hz=650.0, gamma_pot=0.9, tau_pot=3.0, gamma_dep=0.9, tau_dep=2.0,
)


def _llround(x: float) -> int:  # C llround: half away from zero
    r = math.floor(abs(x) + 0.5)
    return int(r) if x >= 0 else -int(r)


def exact_distribution(p, image, q0, T, wta_mode=0, inh_mode=0):
    """Exact law of (final codes, raster) by dynamic programming over the full state."""
    n_in, n_exc = q0.shape
    qmax = 2 ** BITS - 1
    lsb = 2.0 ** -BITS
    dt = p["dt_ms"]
    A = _llround(dt * p["a"] * 65536.0)
    B = _llround(dt * p["b"] * 4294967296.0)
    C = _llround(dt * p["c"] * p["v_spike"] * lsb * 4294967296.0)
    E = _llround(dt * p["c"] * p["i_ext"] * 65536.0)
    Vth, Vreset, Vinit = (_llround(p[k] * 65536.0) for k in ("v_th", "v_reset", "v_init"))

    def lif(v, S):
        return v + A + ((B * v + (1 << 31)) >> 32) + ((C * S + (1 << 15)) >> 16) + E

    p_in = [(p["f_min_hz"] + (p["f_max_hz"] - p["f_min_hz"]) * float(x) / 255.0) * dt * 1e-3 for x in image]

    def P_pot(D):
        return p["gamma_pot"] * math.exp(-D * dt / p["tau_pot"])

    def P_dep(D):
        return p["gamma_dep"] * math.exp(-D * dt / p["tau_dep"])

    state0 = (tuple(int(x) for x in q0.reshape(-1)), (Vinit,) * n_exc, (0,) * n_exc, (-1,) * n_in,
              (-1,) * n_exc, ())
    dist = {state0: 1.0}
    for t in range(T):
        new = defaultdict(float)
        for (q, v, cnt, last_pre, last_post, raster), pr in dist.items():
            for s in itertools.product((0, 1), repeat=n_in):
                ps = 1.0
                for i in range(n_in):
                    ps *= p_in[i] if s[i] else 1.0 - p_in[i]
                if ps == 0.0:
                    continue
                lp = [t if s[i] else last_pre[i] for i in range(n_in)]
                S = [sum(q[i * n_exc + j] for i in range(n_in) if s[i]) for j in range(n_exc)]
                vv, cc, cand = list(v), list(cnt), [False] * n_exc
                for j in range(n_exc):
                    if cc[j] > 0:
                        cc[j] -= 1
                    else:
                        vv[j] = lif(vv[j], S[j])
                        cand[j] = vv[j] > Vth
                if wta_mode == 0:
                    best = None
                    for j in range(n_exc):
                        if cand[j] and (best is None or vv[j] > vv[best]):
                            best = j
                    spikers = [] if best is None else [best]
                else:
                    spikers = [j for j in range(n_exc) if cand[j]]
                for j in spikers:
                    vv[j] = Vreset
                    cc[j] = p["t_ref_steps"]
                if spikers:
                    for j in range(n_exc):
                        if len(spikers) >= 2 or j != spikers[0]:
                            cc[j] = max(cc[j], p["t_inh_steps"])
                            if inh_mode == 0:
                                vv[j] = Vreset
                rbits = sum(1 << j for j in spikers)
                # stochastic STDP trials: LTD first (old last_post), then LTP (last_pre incl. this step)
                trials = []
                for i in range(n_in):
                    if s[i]:
                        for j in range(n_exc):
                            if last_post[j] >= 0:
                                trials.append(("d", i, j, P_dep(t - last_post[j])))
                for W in spikers:
                    for i in range(n_in):
                        if lp[i] >= 0:
                            trials.append(("p", i, W, P_pot(t - lp[i])))
                # every Bernoulli branch, applied in trial order; branches that reach the same codes merge
                qd = {tuple(q): 1.0}
                for kind, i, j, P in trials:
                    k = i * n_exc + j
                    nd = defaultdict(float)
                    for qq, pq in qd.items():
                        if P < 1.0:
                            nd[qq] += pq * (1.0 - P)
                        if P > 0.0:
                            q2 = list(qq)
                            q2[k] = max(q2[k] - 1, 0) if kind == "d" else min(q2[k] + 1, qmax)
                            nd[tuple(q2)] += pq * P
                    qd = nd
                lpost = list(last_post)
                for W in spikers:
                    lpost[W] = t
                for qq, po in qd.items():
                    if po == 0.0:
                        continue
                    key = (qq, tuple(vv), tuple(cc), tuple(lp), tuple(lpost), raster + (rbits,))
                    new[key] += pr * ps * po
        dist = new
    out = defaultdict(float)
    for (q, _v, _c, _lp, _lpo, raster), pr in dist.items():
        out[(q, raster)] += pr
    return dict(out)


def oracle_samples(p, image, q0, T, n, wta_mode=0, inh_mode=0):
    pp = dict(p, wta_mode=wta_mode, inh_mode=inh_mode)
    net = O.OracleNet(N_IN, N_EXC, BITS, pp)
    counts = defaultdict(int)
    for seed in range(n):
        net.set_weights(q0)
        net.present(image, T, seed=seed * 7919 + 13)
        q = tuple(int(x) for x in net.weights().reshape(-1))
        r = tuple(int(w[0]) for w in net.spikes())
        counts[(q, r)] += 1
    return counts


# HOLD inhibition (R7, "inhibitory signal ... for t inh"): an inhibited neuron keeps v.  With
# t_inh = t_ref = 1 a neuron inhibited at t is blocked at t+1 and integrates again at t+2 < T from its HELD
# v (HOLD) or from v_reset (RESET), so the raster law at t = 2 separates the two readings.
PARAMS_HOLD = dict(PARAMS, t_inh_steps=1, t_ref_steps=1)


@pytest.mark.parametrize("wta_mode,inh_mode", [(0, 0), (1, 0), (0, 1), (1, 1)])
def test_bruteforce_matches_oracle_montecarlo(wta_mode, inh_mode):
    prm = PARAMS if inh_mode == 0 else PARAMS_HOLD
    exact = exact_distribution(prm, IMAGE, Q0, T, wta_mode=wta_mode, inh_mode=inh_mode)
    assert abs(sum(exact.values()) - 1.0) < 1e-9
    # the configuration must exercise the rules being pinned
    p_spike = sum(pr for (q, r), pr in exact.items() if any(r))
    p_changed = sum(pr for (q, r), pr in exact.items() if q != tuple(int(x) for x in Q0.reshape(-1)))
    assert p_spike > 0.3 and p_changed > 0.2
    n = 100_000
    mc = oracle_samples(prm, IMAGE, Q0, T, n, wta_mode=wta_mode, inh_mode=inh_mode)
    assert set(mc) <= set(exact), "oracle produced an outcome of probability zero"
    cats = sorted(exact, key=lambda k: -exact[k])
    big = [k for k in cats if exact[k] * n >= 5.0]
    obs = [mc.get(k, 0) for k in big]
    expv = [exact[k] * n for k in big]
    rest_e = n - sum(expv)
    rest_o = n - sum(obs)
    if rest_e >= 5.0:
        obs.append(rest_o)
        expv.append(rest_e)
    chi2 = sum((o - e) ** 2 / e for o, e in zip(obs, expv))
    pval = sst.chi2.sf(chi2, len(obs) - 1)
    assert len(big) >= 20
    assert pval > 1e-3, f"chi2={chi2:.1f} dof={len(obs) - 1} p={pval:.2e}"


def test_bruteforce_detects_a_wrong_phase_order():
    """Sensitivity check: swapping LTD/LTP order or shifting Dt by one changes the law enough
    for the same chi-square to reject it (so the test above has power)."""
    exact = exact_distribution(PARAMS, IMAGE, Q0, T)
    shifted = exact_distribution(dict(PARAMS, tau_dep=PARAMS["tau_dep"] * 1.5), IMAGE, Q0, T)
    n = 100_000
    keys = set(exact) | set(shifted)
    big = [k for k in keys if exact.get(k, 0) * n >= 5.0]
    chi2 = sum((shifted.get(k, 0) * n - exact[k] * n) ** 2 / (exact[k] * n) for k in big)
    assert sst.chi2.sf(chi2, len(big) - 1) < 1e-6


def test_bruteforce_separates_hold_from_reset(wta_mode=0):
    """Power check for the HOLD rows: the exact laws under HOLD and RESET inhibition (same parameters)
    differ enough that 10^5 samples of one reject the other (so a HOLD branch that also resets v fails)."""
    hold = exact_distribution(PARAMS_HOLD, IMAGE, Q0, T, wta_mode=wta_mode, inh_mode=1)
    reset = exact_distribution(PARAMS_HOLD, IMAGE, Q0, T, wta_mode=wta_mode, inh_mode=0)
    n = 100_000
    big = [k for k in hold if hold[k] * n >= 5.0]
    chi2 = sum((reset.get(k, 0) * n - hold[k] * n) ** 2 / (hold[k] * n) for k in big)
    assert sst.chi2.sf(chi2, len(big) - 1) < 1e-6
