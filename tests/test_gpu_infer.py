"""NEXT-1 GPU <-> oracle parity: frozen-weight inference (spike counts), neuron labelling and the class
vote (§III-B, R21-R23).  Integer outputs, so the bar is bit-exact."""
import os

import numpy as np
import pytest

import synthdata
from oracle import oracle as O

pytestmark = pytest.mark.gpu


def _pair(n_in, n_exc, bits, p):
    import paper_conf_date_shelm19_b200 as P
    return P.Network(n_in, n_exc, bits, P.params_from_dict(p)), O.OracleNet(n_in, n_exc, bits, p)


def _random_codes(n_in, n_exc, q_max, seed, density=1.0):
    rng = np.random.default_rng(seed)
    c = rng.integers(0, q_max + 1, size=(n_in, n_exc)).astype(np.uint8)
    if density < 1.0:
        c[rng.random((n_in, n_exc)) > density] = 0
    return c


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("bits", [2, 4, 8])
def test_infer_c1_shape(gpu, mode, bits):
    """784 -> 100, 20 MNIST-shaped images, T = 100, random codes: counts bit-exact; weights untouched."""
    p = O.params({2: "2b", 4: "4b", 8: "8b"}[bits], membrane_mode=mode, init_seed=4, v_spike=3.0)
    g, o = _pair(784, 100, bits, p)
    w = _random_codes(784, 100, (1 << bits) - 1, 11)
    g.set_weights(w); o.set_weights(w)
    imgs = synthdata.images(20, "mnist")
    seeds = synthdata.seeds(20, base_seed=5)
    cg = g.infer(imgs, 100, seeds)
    co = o.infer(imgs, 100, seeds)
    assert co.sum() > 20, "workload must spike"
    assert np.array_equal(cg, co)
    assert np.array_equal(g.weights(), w)
    st = g.infer_stats()
    assert int(st[1]) == int(co.sum())


@pytest.mark.parametrize("mode", [0, 1])
def test_infer_c4_shape_full_size(gpu, mode):
    """784 -> 6400, 2-bit, fashion-shaped, T = 350 (the bench workload) on init weights."""
    p = O.params("2b", membrane_mode=mode, init_seed=1)
    g, o = _pair(784, 6400, 2, p)
    assert np.array_equal(g.weights(), o.weights())
    imgs = synthdata.images(3, "fashion", start=500)
    seeds = synthdata.seeds(3, base_seed=8)
    cg = g.infer(imgs, 350, seeds)
    co = o.infer(imgs, 350, seeds)
    assert co.sum() > 10
    assert np.array_equal(cg, co)


@pytest.mark.parametrize("wta,inh", [(0, 0), (0, 1), (1, 0), (1, 1)])
@pytest.mark.parametrize("n_exc", [1, 31, 33, 65, 400])
def test_infer_modes_and_ragged(gpu, wta, inh, n_exc):
    p = O.params("8b", wta_mode=wta, inh_mode=inh, membrane_mode=1, v_spike=3.0, t_ref_steps=2, t_inh_steps=4)
    g, o = _pair(784, n_exc, 8, p)
    w = _random_codes(784, n_exc, 255, n_exc)
    g.set_weights(w); o.set_weights(w)
    imgs = synthdata.images(6, "mnist", start=40)
    seeds = synthdata.seeds(6, base_seed=13)
    assert np.array_equal(g.infer(imgs, 150, seeds), o.infer(imgs, 150, seeds))


@pytest.mark.parametrize("fmin,fmax", [(5.0, 78.0), (10.0, 312.0), (1000.0, 1000.0)])
def test_infer_high_rates_and_direct_steps(gpu, fmin, fmax):
    """Rates whose steps exceed the ring budget (direct per-column path) and the saturating input."""
    p = O.params("2b", f_min_hz=fmin, f_max_hz=fmax, membrane_mode=0, v_spike=1.0)
    g, o = _pair(784, 500, 2, p)
    w = _random_codes(784, 500, 3, 3, density=0.3)
    g.set_weights(w); o.set_weights(w)
    imgs = synthdata.images(4, "fashion")
    seeds = synthdata.seeds(4, base_seed=21)
    co = o.infer(imgs, 80, seeds)
    assert np.array_equal(g.infer(imgs, 80, seeds), co)


@pytest.mark.parametrize("n_in", [1, 37, 2000])
def test_infer_odd_input_sizes(gpu, n_in):
    p = O.params("4b", f_min_hz=200.0, f_max_hz=400.0, membrane_mode=1, v_spike=4.0)
    g, o = _pair(n_in, 70, 4, p)
    w = _random_codes(n_in, 70, 15, n_in)
    g.set_weights(w); o.set_weights(w)
    rng = np.random.default_rng(n_in)
    imgs = rng.integers(0, 256, size=(5, n_in)).astype(np.uint8)
    seeds = synthdata.seeds(5, base_seed=2)
    assert np.array_equal(g.infer(imgs, 60, seeds), o.infer(imgs, 60, seeds))


def test_infer_persistent_image_loop_and_T_edges(gpu, monkeypatch):
    """More images than CTAs (each CTA strides over images, the producer prefetches across image
    boundaries), T = 1, and T = 0."""
    p = O.params("8b", membrane_mode=0, v_spike=6.0)
    g, o = _pair(784, 100, 8, p)
    imgs = synthdata.images(37, "mnist", start=7)
    seeds = synthdata.seeds(37, base_seed=4)
    monkeypatch.setenv("SNN_INFER_MAX_GRID", "5")
    assert np.array_equal(g.infer(imgs, 90, seeds), o.infer(imgs, 90, seeds))
    assert np.array_equal(g.infer(imgs[:3], 1, seeds[:3]), o.infer(imgs[:3], 1, seeds[:3]))
    assert not g.infer(imgs[:3], 0, seeds[:3]).any()


def test_infer_after_learning_uses_learned_weights(gpu):
    """Learning on the GPU and in the oracle in lockstep, then inference: the inference layout is rebuilt
    from the learned codes (and again after set_weights)."""
    p = O.params("8b", membrane_mode=1, init_seed=9)
    g, o = _pair(784, 100, 8, p)
    imgs = synthdata.images(6, "mnist", start=100)
    seeds = synthdata.seeds(6, base_seed=6)
    assert np.array_equal(g.infer(imgs[3:], 100, seeds[3:]), o.infer(imgs[3:], 100, seeds[3:]))
    for k in range(3):
        g.present(imgs[k], 100, int(seeds[k]))
        o.present(imgs[k], 100, int(seeds[k]))
    assert np.array_equal(g.weights(), o.weights())
    assert np.array_equal(g.infer(imgs[3:], 100, seeds[3:]), o.infer(imgs[3:], 100, seeds[3:]))
    w = _random_codes(784, 100, 255, 1)
    g.set_weights(w); o.set_weights(w)
    assert np.array_equal(g.infer(imgs[3:], 100, seeds[3:]), o.infer(imgs[3:], 100, seeds[3:]))


def test_infer_device_buffers(gpu):
    import torch
    p = O.params("2b", membrane_mode=0)
    g, o = _pair(784, 1600, 2, p)
    imgs = synthdata.images(8, "mnist")
    seeds = synthdata.seeds(8, base_seed=3)
    out = torch.zeros((8, 1600), dtype=torch.int32, device="cuda")
    g.infer(torch.from_numpy(imgs).cuda(), 120, torch.from_numpy(seeds.view(np.int64)).cuda(), out)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy().view(np.uint32), o.infer(imgs, 120, seeds))


def test_label_and_classify_match_oracle(gpu):
    import paper_conf_date_shelm19_b200 as P
    g = P.Network(784, 300, 8, P.preset("8b"))
    rng = np.random.default_rng(0)
    for trial in range(4):
        n, ncls = 500, [10, 3, 64, 1][trial]
        counts = rng.poisson(0.3, size=(n, 300)).astype(np.uint32)
        counts[:, rng.integers(0, 300, size=40)] = 0           # silent neurons -> -1
        classes = rng.integers(0, ncls, size=n).astype(np.int32)
        lab = g.label(counts, classes, ncls)
        assert np.array_equal(lab, O.label(counts, classes, ncls))
        pred = g.classify(counts, lab, ncls)
        assert np.array_equal(pred, O.classify(counts, lab, ncls))
    g2 = P.Network(784, 4, 8, P.preset("8b"))
    gold = [ln.split() for ln in open(os.path.join(os.path.dirname(__file__), "golden", "label_vote_example.txt"))
            if ln.strip() and not ln.startswith("#")]
    lc = np.array([[int(x) for x in r[1:]] for r in gold if r[0] == "label_counts"], np.uint32)
    cl = np.array([int(x) for r in gold if r[0] == "label_classes" for x in r[1:]], np.int32)
    tc = np.array([[int(x) for x in r[1:]] for r in gold if r[0] == "test_counts"], np.uint32)
    lab = g2.label(lc, cl, 3)
    assert lab.tolist() == [0, 1, 1, -1]
    assert g2.classify(tc, lab, 3).tolist() == [1, 0, 0, -1]


def test_full_label_infer_pipeline(gpu):
    """P:88 protocol on synthetic data: learn, label with 'test' images, infer the rest; GPU == oracle
    end to end (counts, labels, predictions)."""
    p = O.params("8b", membrane_mode=1, init_seed=2)
    g, o = _pair(784, 100, 8, p)
    imgs = synthdata.images(40, "mnist", start=3000)
    cls = synthdata.labels(40, start=3000).astype(np.int32)
    seeds = synthdata.seeds(40, base_seed=17)
    for k in range(10):
        g.present(imgs[k], 100, int(seeds[k]))
        o.present(imgs[k], 100, int(seeds[k]))
    cg = g.infer(imgs[10:], 100, seeds[10:])
    co = o.infer(imgs[10:], 100, seeds[10:])
    assert np.array_equal(cg, co)
    lg = g.label(cg[:15], cls[10:25], 10)
    assert np.array_equal(lg, O.label(co[:15], cls[10:25], 10))
    assert np.array_equal(g.classify(cg[15:], lg, 10), O.classify(co[15:], lg, 10))


def test_infer_rejects_bad_arguments(gpu):
    import paper_conf_date_shelm19_b200 as P
    g = P.Network(784, 100, 8, P.preset("8b"))
    imgs = synthdata.images(2, "mnist")
    seeds = synthdata.seeds(2)
    with pytest.raises(P.SnnError):
        g.infer(imgs, 70000, seeds)
    with pytest.raises(P.SnnError):
        g.label(np.zeros((2, 100), np.uint32), np.array([0, 5], np.int32), 3)
    with pytest.raises(P.SnnError):
        g.classify(np.zeros((2, 100), np.uint32), np.full(100, 7, np.int32), 3)
    big = P.Network(784, 8000, 2, P.preset("2b"))
    with pytest.raises(P.SnnError):
        big.infer(imgs, 10, seeds)
