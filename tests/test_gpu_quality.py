"""NEXT-1 analysis half: qualitative checks of learning on the synthetic
proxy (the accuracy figures themselves need the real datasets: "parity unpinned").  Runs the P:88 protocol
entirely in the CUDA library (train, label with a labelling set, classify an evaluation set).

* Reading R6b: with the winner's refractory period shorter than the others' inhibition
  (t_ref 5 < t_inh 10) the winner restarts ahead of everyone after each spike and one neuron soon wins every
  image (the vote degenerates to one class, error 0.9 = chance); with t_ref = t_inh no column gets a head
  start and the error of the 784 -> 400 8-bit stochastic network is clearly below chance.
* P:104 Table II "Bit truncation shows the lowest accuracy" / Q0.2 baseline 9.6 %: at 2 bits the
  deterministic rule's eq.(4)(5) steps (<= 0.04 LSB) truncate to zero, so the codes never move (the
  Fig. 6(b)-style conductance histogram stays the initial one), while the stochastic rule moves them.
"""
import numpy as np
import pytest

import synthdata

pytestmark = pytest.mark.gpu


def _train(bits, preset, overrides, n_train=1000, n_lab=500, n_eval=500):
    import paper_conf_date_shelm19_b200 as P
    from paper_conf_date_shelm19_b200.schedule import Phase, run_schedule
    tr, trs = synthdata.images(n_train, "mnist"), synthdata.seeds(n_train, 1)
    li, lc, ls = synthdata.images(n_lab, "mnist", start=50000), synthdata.labels(n_lab, 50000), synthdata.seeds(n_lab, 2)
    ei, ec, es = synthdata.images(n_eval, "mnist", start=60000), synthdata.labels(n_eval, 60000), synthdata.seeds(n_eval, 3)
    init = P.Network(784, 400, bits, P.preset(preset, **overrides)).weights()
    curve, net = run_schedule(784, 400, bits, [Phase(preset, 350, n_train, dict(overrides))], tr, trs, li, lc, ls,
                              ei, ec, es, eval_every=n_train)
    counts = net.infer(ei, 350, es)
    return curve[-1].error, int((counts.sum(axis=0) > 0).sum()), init, net.weights()


def test_head_start_reading_collapses_and_equal_refractory_learns(gpu):
    err_default, active_default, _, _ = _train(8, "8b", dict(t_ref_steps=5, t_inh_steps=10))
    assert err_default >= 0.89 and active_default <= 2            # one neuron wins every image
    err, active, _, _ = _train(8, "8b", dict(t_ref_steps=10, t_inh_steps=10))
    assert err <= 0.8 and active >= 300                            # chance is 0.9


def test_q02_truncation_never_learns_stochastic_does(gpu):
    ov = dict(t_ref_steps=10, t_inh_steps=10)
    _, _, init, w_det = _train(2, "2b", dict(ov, stdp_mode=1, rounding=0), n_train=300, n_lab=50, n_eval=50)
    assert np.array_equal(w_det, init)                             # eq.(4)(5) <= 0.04 LSB truncate to 0
    _, _, init, w_sto = _train(2, "2b", dict(ov, stdp_mode=0), n_train=300, n_lab=50, n_eval=50)
    assert not np.array_equal(w_sto, init)
    h0, h1 = np.bincount(init.ravel(), minlength=4), np.bincount(w_sto.ravel(), minlength=4)
    assert h1[3] > h0[3]                                           # LTP drives the active synapses to G_max
