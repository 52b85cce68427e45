"""NEXT-4 GPU <-> oracle parity: the Fig. 4 sparse recurrent workload (R24-R26).
Integer outputs (spike counts, rasters): bit-exact."""
import numpy as np
import pytest

import synthdata
from oracle import oracle as O

pytestmark = pytest.mark.gpu


def _run_both(bits, p, n_lif, n_syn, n_trials, T, kind="fashion", recurrent=True, seed=1):
    import paper_conf_date_shelm19_b200 as P
    g = P.Network(784, 64, bits, P.params_from_dict(p))
    o = O.OracleNet(784, 64, bits, p)
    off, tgt, q = synthdata.sparse_graph(784, n_lif, n_syn, bits=bits, seed=seed, recurrent=recurrent)
    imgs = synthdata.images(n_trials, kind, start=seed)
    seeds = synthdata.seeds(n_trials, base_seed=seed + 3)
    wl = (n_lif + 31) // 32
    rg = np.zeros((n_trials, T, wl), np.uint32)
    cg = g.sparse_run(n_lif, off, tgt, q, imgs, T, seeds, raster=rg)
    co, ro = o.sparse_run(n_lif, off, tgt, q, imgs, T, seeds, raster=True)
    return cg, rg, co, ro, g


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("bits", [2, 4, 8])
def test_sparse_fig4_shape(gpu, mode, bits):
    """10^3 LIF neurons, 10^4 synapses, 5-78 Hz drive strong enough to spike; rasters bit-exact."""
    vs = 32.0 / (2.0 ** -bits * ((1 << bits) - 1) / 2)          # I ~ 32 mV-units per unit of mean code flow
    p = O.params({2: "2b", 4: "4b", 8: "8b"}[bits], membrane_mode=mode, v_spike=vs,
                 f_min_hz=5.0, f_max_hz=78.0)
    cg, rg, co, ro, g = _run_both(bits, p, 1000, 10000, 6, 200)
    assert co.sum() > 50
    assert np.array_equal(cg, co)
    assert np.array_equal(rg, ro)
    st = g.sparse_stats()
    assert int(st[1]) == int(co.sum())


@pytest.mark.parametrize("n_lif,n_syn", [(1, 50), (33, 400), (700, 20000), (3000, 30000)])
def test_sparse_sizes_and_dense_graphs(gpu, n_lif, n_syn):
    p = O.params("8b", membrane_mode=1, v_spike=30.0, f_min_hz=20.0, f_max_hz=200.0, t_ref_steps=2)
    cg, rg, co, ro, _ = _run_both(8, p, n_lif, n_syn, 3, 120, seed=n_lif)
    assert np.array_equal(cg, co)
    assert np.array_equal(rg, ro)


def test_sparse_feedforward_and_many_trials(gpu):
    p = O.params("4b", membrane_mode=0, v_spike=40.0, f_min_hz=5.0, f_max_hz=78.0)
    cg, rg, co, ro, _ = _run_both(4, p, 1000, 10000, 700, 40, kind="mnist", recurrent=False, seed=9)
    assert np.array_equal(cg, co)


def test_sparse_rejects_bad_graph(gpu):
    import paper_conf_date_shelm19_b200 as P
    g = P.Network(784, 64, 4, P.preset("4b"))
    off, tgt, q = synthdata.sparse_graph(784, 10, 100, bits=4)
    imgs, seeds = synthdata.images(1), synthdata.seeds(1)
    bad = q.copy(); bad[0] = 16
    with pytest.raises(P.SnnError):
        g.sparse_run(10, off, tgt, bad, imgs, 5, seeds)
    badt = tgt.copy(); badt[3] = 10
    with pytest.raises(P.SnnError):
        g.sparse_run(10, off, badt, q, imgs, 5, seeds)
    bado = off.copy(); bado[5] = bado[6] + 1
    with pytest.raises(P.SnnError):
        g.sparse_run(10, bado, tgt, q, imgs, 5, seeds)
