"""Pins of the oracle's NEXT-1 functions (labelling + inference with frozen weights, §III-B;
readings DESIGN.md R21-R23).  No GPU; no expected value comes from the CUDA path."""
import math
import os

import numpy as np
import pytest

from oracle import oracle as O
import synthdata

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "label_vote_example.txt")


def _golden():
    d = {"label_counts": [], "test_counts": []}
    for line in open(GOLDEN):
        if not line.strip() or line.startswith("#"):
            continue
        k, *v = line.split()
        v = [int(x) for x in v]
        if k in d and isinstance(d[k], list) and k.endswith("counts"):
            d[k].append(v)
        else:
            d[k] = v
    return d


def test_label_and_vote_hand_worked_example():
    g = _golden()
    lc = np.array(g["label_counts"], np.uint32)
    labels = O.label(lc, g["label_classes"], g["n_classes"][0])
    assert labels.tolist() == g["labels"]
    pred = O.classify(np.array(g["test_counts"], np.uint32), labels, g["n_classes"][0])
    assert pred.tolist() == g["pred"]


def test_label_invariances():
    """R22 depends on per-class MEAN responses: image order and duplicating the labelling set do not
    change labels; renaming classes by a permutation renames the labels."""
    rng = np.random.default_rng(5)
    counts = rng.poisson(0.7, size=(60, 40)).astype(np.uint32)
    classes = rng.integers(0, 6, size=60).astype(np.int32)
    base = O.label(counts, classes, 6)
    perm = rng.permutation(60)
    assert np.array_equal(O.label(counts[perm], classes[perm], 6), base)
    assert np.array_equal(O.label(np.vstack([counts, counts]), np.concatenate([classes, classes]), 6), base)
    pi = rng.permutation(6).astype(np.int32)
    relab = O.label(counts, pi[classes], 6)
    # ties -> lowest class index is not permutation-invariant; compare where the best class is unique
    for j in range(40):
        r = np.array([counts[classes == c, j].sum() / max(1, (classes == c).sum()) for c in range(6)])
        if r.max() == 0:
            assert base[j] == -1 and relab[j] == -1
        elif (r == r.max()).sum() == 1:
            assert relab[j] == pi[base[j]]


def test_label_single_class_responder_and_ties():
    counts = np.array([[0, 5, 1], [0, 0, 1], [0, 0, 1], [0, 0, 1]], np.uint32)
    classes = np.array([2, 1, 0, 3], np.int32)
    # neuron 0 silent -> -1; neuron 1 responds only to class 2; neuron 2 equal mean everywhere -> lowest (0)
    assert O.label(counts, classes, 4).tolist() == [-1, 2, 0]
    # a class with no labelling image never wins
    assert O.label(np.array([[1]], np.uint32), np.array([3], np.int32), 5).tolist() == [3]


def test_classify_one_hot_design_is_perfect():
    """Neurons that fire only for their own class classify every image correctly (R23)."""
    n_classes, per = 10, 7
    labels = np.repeat(np.arange(n_classes, dtype=np.int32), per)
    rng = np.random.default_rng(2)
    truth = rng.integers(0, n_classes, size=200)
    counts = np.zeros((200, n_classes * per), np.uint32)
    for k, c in enumerate(truth):
        counts[k, c * per:(c + 1) * per] = rng.integers(1, 4, size=per)
        counts[k, rng.integers(0, n_classes * per)] += 0   # no cross-class spikes
    assert np.array_equal(O.classify(counts, labels, n_classes), truth)
    assert O.classify(np.zeros((3, n_classes * per), np.uint32), labels, n_classes).tolist() == [-1] * 3


def test_classify_mean_not_sum():
    # class 0 has 1 neuron (3 spikes, mean 3); class 1 has 4 neurons (1 spike each, sum 4, mean 1)
    labels = np.array([0, 1, 1, 1, 1], np.int32)
    assert O.classify(np.array([[3, 1, 1, 1, 1]], np.uint32), labels, 2).tolist() == [0]


def test_label_rejects_bad_class():
    with pytest.raises(O.OracleError):
        O.label(np.zeros((1, 2), np.uint32), np.array([4], np.int32), 4)


@pytest.mark.parametrize("mode", [0, 1])
def test_infer_equals_learning_with_gamma_zero(mode):
    """With gamma_pot = gamma_dep = 0 STDP never changes a code (eqs.(6)(7)), so a learning presentation
    and a frozen-weight presentation (R21) give the same raster; infer never changes the weights."""
    p = O.params("8b", membrane_mode=mode, init_seed=3, v_spike=6.0)
    imgs = synthdata.images(3, "mnist")
    seeds = synthdata.seeds(3, base_seed=9)
    a = O.OracleNet(784, 50, 8, p)
    w0 = a.weights()
    counts = a.infer(imgs, 120, seeds)
    assert np.array_equal(a.weights(), w0)
    b = O.OracleNet(784, 50, 8, O.params("8b", membrane_mode=mode, init_seed=3, v_spike=6.0,
                                         gamma_pot=0.0, gamma_dep=0.0))
    for k in range(3):
        b.present(imgs[k], 120, int(seeds[k]))
        r = O.unpack_bits(b.spikes(), 50)
        assert np.array_equal(r.sum(axis=0).astype(np.uint32), counts[k])
    assert counts.sum() > 0
    # learning ON (8-bit row) changes the weights and (generally) the spikes; infer must not
    c = O.OracleNet(784, 50, 8, p)
    c.present(imgs[0], 120, int(seeds[0]))
    assert not np.array_equal(c.weights(), w0)


def _k_first(I, v0, p=O.BASE):
    a, b, c, vth, dt = p["a"], p["b"], p["c"], p["v_th"], p["dt_ms"]
    lam, vinf = 1.0 + b * dt, -(a + c * I) / b
    return math.floor(math.log((vinf - vth) / (vinf - v0)) / math.log(lam)) + 1


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("qval,T", [(1, 350), (2, 100)])
def test_infer_counts_closed_form(mode, qval, T):
    """Saturating input (p = 1): I = v_spike LSB 784 q (eq.(3)).  Identical columns: the lowest index
    always wins (R7), is refractory t_ref steps, then integrates from v_reset; everyone else is reset and
    held t_inh > t_ref steps, so neuron 0 spikes at s1 = k(I, -70) - 1 and every t_ref + k(I, v_reset)
    steps after (eqs.(1)(2) closed form under forward Euler)."""
    p = O.params("8b", v_spike=1.0, f_min_hz=1000.0, f_max_hz=1000.0, membrane_mode=mode)
    net = O.OracleNet(784, 5, 8, p)
    net.set_weights(np.full((784, 5), qval, np.uint8))
    counts = net.infer(np.full((1, 784), 200, np.uint8), T, [77])
    I = 784 * qval / 256.0
    s1 = _k_first(I, -70.0) - 1
    period = p["t_ref_steps"] + _k_first(I, p["v_reset"])
    expect = 1 + (T - 1 - s1) // period
    assert counts[0].tolist() == [expect, 0, 0, 0, 0]
