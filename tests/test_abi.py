"""C-ABI checks that need no GPU: the in-tree library loads, exports every function that
include/snn.h declares, validates parameters before touching CUDA, and its parameter block has
the layout DESIGN.md §3.1 documents (the oracle's hand-written copy must agree byte for byte)."""
import ctypes
import os
import re

import pytest

import paper_conf_date_shelm19_b200 as P
from paper_conf_date_shelm19_b200 import snn as S
from oracle import oracle as O

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _header_functions():
    src = open(os.path.join(ROOT, "include", "snn.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(snn_[a-z_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    L = S.lib()
    declared = _header_functions()
    assert len(declared) >= 20
    for name in declared:
        assert hasattr(L, name), name
    assert sorted(S.EXPORTS) == declared


def test_library_is_sm100a():
    out = os.popen(f"/usr/local/cuda/bin/cuobjdump -lelf {S.LIB_PATH} 2>&1").read()
    assert "sm_100a" in out


def test_params_layout_matches_oracle_copy():
    assert ctypes.sizeof(S.SnnParams) == ctypes.sizeof(O.OracleParams)
    for (n1, t1), (n2, t2) in zip(S.SnnParams._fields_, O.OracleParams._fields_):
        assert n1 == n2 or (n1, n2) == ("engine", "reserved0")   # the oracle has one semantics, no engines
        assert getattr(S.SnnParams, n1).offset == getattr(O.OracleParams, n2).offset
        assert ctypes.sizeof(t1) == ctypes.sizeof(t2)


TABLE_I = {  # gamma_pot tau_pot gamma_dep tau_dep f_max f_min
    "2b": (0.2, 20, 0.2, 10, 22, 1), "4b": (0.3, 30, 0.3, 10, 22, 1), "8b": (0.5, 30, 0.5, 10, 22, 1),
    "16b": (0.9, 30, 0.9, 10, 22, 1), "hf": (0.3, 80, 0.2, 5, 78, 5),
}


@pytest.mark.parametrize("name", sorted(TABLE_I))
def test_presets_transcribe_table_I(name):
    p = P.preset(name)
    assert (p.gamma_pot, p.tau_pot, p.gamma_dep, p.tau_dep, p.f_max_hz, p.f_min_hz) == TABLE_I[name]
    # P:90 §III-D
    assert (p.a, p.b, p.c, p.v_th, p.v_reset, p.v_init) == (-6.77, -0.0989, 0.314, -60.2, -74.7, -70.0)
    assert (p.alpha_p, p.beta_p, p.alpha_d, p.beta_d, p.g_max, p.g_min) == (0.01, 3.0, 0.005, 3.0, 1.0, 0.0)


def test_presets_agree_with_oracle_presets():
    for name in TABLE_I:
        a = P.preset(name).as_dict()
        b = O.params(name)
        a.pop("engine")
        for k in a:
            assert a[k] == pytest.approx(b[k]), (name, k)


@pytest.mark.parametrize("bad", [dict(gamma_pot=1.5), dict(tau_dep=0.0), dict(f_max_hz=2000.0), dict(wta_mode=3),
                                 dict(g_min=0.1), dict(rounding=7), dict(tau_pot=1e6), dict(cluster_size=17)])
def test_invalid_params_rejected_before_cuda(bad):
    with pytest.raises(P.SnnError) as e:
        P.Network(784, 10, 8, P.preset("8b", **bad))
    assert e.value.rc == S.SNN_EINVAL


@pytest.mark.parametrize("bits", [0, 1, 3, 12, 24, 64])
def test_invalid_bits_rejected(bits):
    with pytest.raises(P.SnnError) as e:
        P.Network(784, 10, bits, P.preset("8b"))
    assert e.value.rc == S.SNN_EINVAL


@pytest.mark.parametrize("bad", [dict(membrane_mode=1), dict(rounding=0), dict(rounding=2)])
def test_fp32_conductance_mode_constraints(bad):
    """bits = 32 (R28): binary32 conductance needs fp32 membranes and round-to-nearest; rejected before CUDA."""
    with pytest.raises(P.SnnError) as e:
        P.Network(784, 10, 32, P.preset("16b", **bad))
    assert e.value.rc == S.SNN_EINVAL


def test_null_arguments():
    L = S.lib()
    assert L.snn_create(784, 10, 8, None, None) == S.SNN_EINVAL
    assert L.snn_present(None, None, 10, 1) == S.SNN_EINVAL
    assert L.snn_get_weights(None, None, 0) == S.SNN_EINVAL
    assert L.snn_destroy(None) == S.SNN_OK
    assert isinstance(L.snn_last_error(), bytes)


def test_no_gpu_fails_loudly():
    """Without a device the product path errors (SNN_ECUDA); there is no CPU fallback."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(P.SnnError) as e:
        P.Network(784, 100, 8)
    assert e.value.rc == S.SNN_ECUDA


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_date_shelm19_b200")
    bad = re.compile(r"(^\s*(from|import)\s+oracle)|liboracle|snn_oracle|#include\s*[<\"][^>\"]*oracle", re.M)
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".h", ".cuh", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not bad.search(txt), f
