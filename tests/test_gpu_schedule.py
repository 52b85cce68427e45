"""NEXT-3 (frequency-control schedule, P:87 / P:94): the GPU driver's whole run -- phase
changes with carried-over codes, periodic labelling + evaluation -- equals the same protocol run on the
CPU oracle: codes after every phase and every point of the error curve, bit for bit."""
import numpy as np
import pytest

import synthdata
from oracle import oracle as O


def _oracle_schedule(n_in, n_exc, bits, phases, tr, trs, li, lc, ls, ei, ec, es, every, n_classes=10):
    net, seen, curve = None, 0, []
    for pi, ph in enumerate(phases):
        new = O.OracleNet(n_in, n_exc, bits, O.params(ph.preset, **ph.overrides))
        if net is not None:
            new.set_weights(net.weights())
        net = new
        done = 0
        while done < ph.n_images:
            nb = min(every - (seen % every), ph.n_images - done)
            for k in range(seen, seen + nb):
                net.present(tr[k], ph.T, int(trs[k]))
            seen += nb
            done += nb
            if seen % every == 0:
                labels = O.label(net.infer(li, ph.T, ls), lc, n_classes)
                pred = O.classify(net.infer(ei, ph.T, es), labels, n_classes)
                curve.append((seen, float(np.mean(pred != ec)), pi))
    return curve, net


@pytest.mark.gpu
def test_schedule_matches_oracle(gpu):
    from paper_conf_date_shelm19_b200 import schedule as S
    hf = {k: O.TABLE_I["hf"][k] for k in ("f_min_hz", "f_max_hz", "gamma_pot", "tau_pot", "gamma_dep", "tau_dep")}
    phases = [S.Phase("8b", 60, 6, dict(membrane_mode=1)),
              S.Phase("8b", 60, 6, dict(hf, membrane_mode=1)),
              S.Phase("8b", 30, 6, dict(hf, membrane_mode=1))]
    n = 18
    tr = synthdata.images(n, "mnist", start=50)
    trs = synthdata.seeds(n, base_seed=31)
    li, lc, ls = synthdata.images(10, "mnist", start=900), synthdata.labels(10, start=900), synthdata.seeds(10, 32)
    ei, ec, es = synthdata.images(10, "mnist", start=950), synthdata.labels(10, start=950), synthdata.seeds(10, 33)
    curve, net = S.run_schedule(784, 100, 8, phases, tr, trs, li, lc, ls, ei, ec, es, eval_every=6)
    oc, onet = _oracle_schedule(784, 100, 8, phases, tr, trs, li, lc, ls, ei, ec, es, every=6)
    assert [(p.images, p.error, p.phase) for p in curve] == oc
    assert np.array_equal(net.weights(), onet.weights())
    assert [p.sim_ms for p in curve] == [360.0, 720.0, 900.0]


def test_paper_phases_are_table_I_rows():
    from paper_conf_date_shelm19_b200 import schedule as S
    ph = S.paper_phases(10, 20, 30)
    assert [p.T for p in ph] == [500, 500, 100]                      # 500 ms -> 100 ms
    assert ph[0].overrides == {}
    for p in ph[1:]:                                                 # Table I "high frequency" row
        assert (p.overrides["f_min_hz"], p.overrides["f_max_hz"]) == (5.0, 78.0)
        assert (p.overrides["tau_pot"], p.overrides["tau_dep"]) == (80.0, 5.0)
        assert (p.overrides["gamma_pot"], p.overrides["gamma_dep"]) == (0.3, 0.2)
