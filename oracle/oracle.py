"""ctypes binding of the CPU ORACLE (oracle/liboracle.so).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs, never by the product package.  It shares no code
with paper_conf_date_shelm19_b200/; the parameter presets below are transcribed from the
paper's Table I independently of the C library's snn_params_preset.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")

ORACLE_RASTER_INPUT = 1
ORACLE_KEEP_STATE = 2
ORACLE_NO_LEARN = 8


class OracleParams(ctypes.Structure):
    # Layout duplicated by hand from DESIGN.md §3.1 (not generated from include/snn.h).
    _fields_ = [
        ("a", ctypes.c_double), ("b", ctypes.c_double), ("c", ctypes.c_double),
        ("v_th", ctypes.c_double), ("v_reset", ctypes.c_double), ("v_init", ctypes.c_double),
        ("dt_ms", ctypes.c_double), ("v_spike", ctypes.c_double), ("i_ext", ctypes.c_double),
        ("t_ref_steps", ctypes.c_int32), ("t_inh_steps", ctypes.c_int32),
        ("wta_mode", ctypes.c_int32), ("inh_mode", ctypes.c_int32),
        ("f_min_hz", ctypes.c_double), ("f_max_hz", ctypes.c_double),
        ("stdp_mode", ctypes.c_int32), ("rounding", ctypes.c_int32),
        ("t_ltp_steps", ctypes.c_int32), ("membrane_mode", ctypes.c_int32),
        ("gamma_pot", ctypes.c_double), ("tau_pot", ctypes.c_double),
        ("gamma_dep", ctypes.c_double), ("tau_dep", ctypes.c_double),
        ("alpha_p", ctypes.c_double), ("beta_p", ctypes.c_double),
        ("alpha_d", ctypes.c_double), ("beta_d", ctypes.c_double),
        ("g_min", ctypes.c_double), ("g_max", ctypes.c_double),
        ("frac_bits", ctypes.c_int32), ("init_mode", ctypes.c_int32),
        ("init_seed", ctypes.c_uint64),
        ("cluster_size", ctypes.c_int32), ("reserved0", ctypes.c_int32),
    ]


# P:90 §III-D: "V th is -60.2, V reset is -74.7, a is -6.77, b is -0.0989 and c is 0.314",
# "Initial membrane potential ... is -70.0".  Unstated values are DESIGN.md readings (R1, R3, R6, R7, R16).
BASE = dict(
    a=-6.77, b=-0.0989, c=0.314, v_th=-60.2, v_reset=-74.7, v_init=-70.0,
    dt_ms=1.0, v_spike=2.0, i_ext=0.0,
    t_ref_steps=5, t_inh_steps=10, wta_mode=0, inh_mode=0,
    f_min_hz=1.0, f_max_hz=22.0,
    stdp_mode=0, rounding=1, t_ltp_steps=20, membrane_mode=0,
    gamma_pot=0.5, tau_pot=30.0, gamma_dep=0.5, tau_dep=10.0,
    alpha_p=0.01, beta_p=3.0, alpha_d=0.005, beta_d=3.0, g_min=0.0, g_max=1.0,
    frac_bits=0, init_mode=0, init_seed=1, cluster_size=0, reserved0=0,
)

# Table I: columns alpha_P beta_P alpha_D beta_D G_max G_min gamma_pot tau_pot gamma_dep tau_dep f_max f_min
TABLE_I = {
    "2b": dict(gamma_pot=0.2, tau_pot=20.0, gamma_dep=0.2, tau_dep=10.0, f_max_hz=22.0, f_min_hz=1.0),
    "4b": dict(gamma_pot=0.3, tau_pot=30.0, gamma_dep=0.3, tau_dep=10.0, f_max_hz=22.0, f_min_hz=1.0),
    "8b": dict(gamma_pot=0.5, tau_pot=30.0, gamma_dep=0.5, tau_dep=10.0, f_max_hz=22.0, f_min_hz=1.0),
    "16b": dict(alpha_p=0.01, beta_p=3.0, alpha_d=0.005, beta_d=3.0, g_max=1.0, g_min=0.0,
                gamma_pot=0.9, tau_pot=30.0, gamma_dep=0.9, tau_dep=10.0, f_max_hz=22.0, f_min_hz=1.0),
    "hf": dict(alpha_p=0.01, beta_p=3.0, alpha_d=0.005, beta_d=3.0, g_max=1.0, g_min=0.0,
               gamma_pot=0.3, tau_pot=80.0, gamma_dep=0.2, tau_dep=5.0, f_max_hz=78.0, f_min_hz=5.0),
}


def params(preset: str = "8b", **overrides) -> dict:
    p = dict(BASE)
    p.update(TABLE_I[preset])
    for k, v in overrides.items():
        if k not in p:
            raise KeyError(k)
        p[k] = v
    return p


def to_struct(p: dict) -> OracleParams:
    s = OracleParams()
    for name, _ in OracleParams._fields_:
        setattr(s, name, p[name])
    return s


_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"oracle library not built: {_LIB_PATH} (run __graft_entry__.build())")
        L = ctypes.CDLL(_LIB_PATH)
        u32p = ctypes.POINTER(ctypes.c_uint32)
        L.oracle_philox4x32_10.argtypes = [u32p, u32p, u32p]
        L.oracle_create.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.POINTER(OracleParams),
                                    ctypes.POINTER(ctypes.c_void_p)]
        L.oracle_destroy.argtypes = [ctypes.c_void_p]
        L.oracle_present.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int, ctypes.c_uint64]
        L.oracle_present_ex.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int, ctypes.c_uint64,
                                        ctypes.c_int, ctypes.c_int]
        L.oracle_get_weights.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
        L.oracle_set_weights.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
        L.oracle_get_spikes.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t]
        L.oracle_get_input_raster.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t]
        L.oracle_state_bytes.argtypes = [ctypes.c_void_p]
        L.oracle_state_bytes.restype = ctypes.c_size_t
        L.oracle_get_state.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t]
        L.oracle_set_state.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t]
        L.oracle_get_stats.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
        L.oracle_q_max.argtypes = [ctypes.c_void_p]
        L.oracle_lut.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p, ctypes.c_int]
        L.oracle_lif_step_fp32.argtypes = [ctypes.c_void_p, ctypes.c_float, ctypes.c_int32]
        L.oracle_lif_step_fp32.restype = ctypes.c_float
        L.oracle_lif_step_fixed.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32]
        L.oracle_lif_step_fp32g.argtypes = [ctypes.c_void_p, ctypes.c_float, ctypes.c_float]
        L.oracle_lif_step_fp32g.restype = ctypes.c_float
        L.oracle_exp_recipe.argtypes = [ctypes.c_void_p, ctypes.c_double]
        L.oracle_exp_recipe.restype = ctypes.c_double
        L.oracle_dg.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_float]
        L.oracle_dg.restype = ctypes.c_double
        L.oracle_lif_step_fixed.restype = ctypes.c_int32
        L.oracle_infer.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p,
                                   ctypes.c_void_p]
        L.oracle_label.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int,
                                   ctypes.c_void_p]
        L.oracle_sparse_run.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                                        ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p,
                                        ctypes.c_void_p, ctypes.c_void_p]
        L.oracle_classify.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int,
                                      ctypes.c_void_p]
        _lib = L
    return _lib


def philox4x32_10(ctr, key):
    c = (ctypes.c_uint32 * 4)(*[int(x) & 0xFFFFFFFF for x in ctr])
    k = (ctypes.c_uint32 * 2)(*[int(x) & 0xFFFFFFFF for x in key])
    o = (ctypes.c_uint32 * 4)()
    lib().oracle_philox4x32_10(c, k, o)
    return [int(x) for x in o]


def _ptr(a: np.ndarray) -> ctypes.c_void_p:
    return ctypes.c_void_p(a.ctypes.data)


class OracleError(RuntimeError):
    def __init__(self, rc, what):
        super().__init__(f"{what} failed rc={rc}")
        self.rc = rc


class OracleNet:
    """One network (n_in -> n_exc, `bits`-bit codes) simulated by the CPU oracle."""

    def __init__(self, n_in: int, n_exc: int, bits: int, p: dict):
        self.n_in, self.n_exc, self.bits, self.p = n_in, n_exc, bits, dict(p)
        self._h = ctypes.c_void_p()
        self._ps = to_struct(p)
        rc = lib().oracle_create(n_in, n_exc, bits, ctypes.byref(self._ps), ctypes.byref(self._h))
        if rc != 0:
            raise OracleError(rc, "oracle_create")
        self.last_T = 0

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value:
            lib().oracle_destroy(h)
            self._h = ctypes.c_void_p()

    def _check(self, rc, what):
        if rc != 0:
            raise OracleError(rc, what)

    @property
    def q_max(self) -> int:
        return int(lib().oracle_q_max(self._h))

    def present(self, image: np.ndarray, T: int, seed: int):
        img = np.ascontiguousarray(image, dtype=np.uint8).reshape(-1)
        assert img.size == self.n_in
        self._check(lib().oracle_present(self._h, _ptr(img), T, seed), "oracle_present")
        self.last_T = T

    def present_ex(self, inp: np.ndarray, T: int, seed: int, flags: int = 0, t0: int = 0):
        if flags & ORACLE_RASTER_INPUT:
            arr = np.ascontiguousarray(inp, dtype=np.uint32).reshape(-1)
            assert arr.size >= T * ((self.n_in + 31) // 32)
        else:
            arr = np.ascontiguousarray(inp, dtype=np.uint8).reshape(-1)
            assert arr.size == self.n_in
        self._check(lib().oracle_present_ex(self._h, _ptr(arr), T, seed, flags, t0), "oracle_present_ex")
        self.last_T = T

    def present_raster(self, raster: np.ndarray, T: int, seed: int, keep_state=False, t0=0):
        flags = ORACLE_RASTER_INPUT | (ORACLE_KEEP_STATE if keep_state else 0)
        self.present_ex(raster, T, seed, flags, t0)

    @property
    def code_dtype(self):
        """uint8 codes (<= 8 bits), uint16 codes (16 bits), binary32 conductance (32 bits, R28)"""
        return np.float32 if self.bits == 32 else (np.uint16 if self.bits > 8 else np.uint8)

    def weights(self) -> np.ndarray:
        out = np.empty((self.n_in, self.n_exc), dtype=self.code_dtype)
        self._check(lib().oracle_get_weights(self._h, _ptr(out)), "oracle_get_weights")
        return out

    def set_weights(self, codes: np.ndarray):
        c = np.ascontiguousarray(codes, dtype=self.code_dtype).reshape(self.n_in, self.n_exc)
        self._check(lib().oracle_set_weights(self._h, _ptr(c)), "oracle_set_weights")

    def spikes(self) -> np.ndarray:
        we = (self.n_exc + 31) // 32
        out = np.zeros((max(self.last_T, 0), we), dtype=np.uint32)
        self._check(lib().oracle_get_spikes(self._h, _ptr(out), out.size), "oracle_get_spikes")
        return out

    def input_raster(self) -> np.ndarray:
        wi = (self.n_in + 31) // 32
        out = np.zeros((max(self.last_T, 0), wi), dtype=np.uint32)
        self._check(lib().oracle_get_input_raster(self._h, _ptr(out), out.size), "oracle_get_input_raster")
        return out

    def state_bytes(self) -> int:
        return int(lib().oracle_state_bytes(self._h))

    def state(self) -> np.ndarray:
        out = np.zeros(self.state_bytes() // 4, dtype=np.int32)
        self._check(lib().oracle_get_state(self._h, _ptr(out), out.nbytes), "oracle_get_state")
        return out

    def set_state(self, blob: np.ndarray):
        b = np.ascontiguousarray(blob, dtype=np.int32)
        self._check(lib().oracle_set_state(self._h, _ptr(b), b.nbytes), "oracle_set_state")

    def stats(self) -> np.ndarray:
        out = np.zeros(8, dtype=np.uint64)
        self._check(lib().oracle_get_stats(self._h, _ptr(out)), "oracle_get_stats")
        return out

    def lut(self, which: int) -> np.ndarray:
        out = np.zeros(8192, dtype=np.uint64)
        n = lib().oracle_lut(self._h, which, _ptr(out), out.size)
        if n < 0:
            raise OracleError(n, "oracle_lut")
        return out[:n].copy()

    def lif_step_fp32(self, v: float, S: int) -> float:
        return float(lib().oracle_lif_step_fp32(self._h, ctypes.c_float(v), int(S)))

    def lif_step_fixed(self, v: int, S: int) -> int:
        return int(lib().oracle_lif_step_fixed(self._h, int(v), int(S)))

    def lif_step_fp32g(self, v: float, Sg: float) -> float:
        """32-bit arm (R28): LIF update on the binary32 conductance sum."""
        return float(lib().oracle_lif_step_fp32g(self._h, ctypes.c_float(v), ctypes.c_float(Sg)))

    def exp_recipe(self, y: float) -> float:
        """R28's binary64 e^y recipe."""
        return float(lib().oracle_exp_recipe(self._h, float(y)))

    def dg(self, depress: bool, G: float) -> float:
        """eqs.(4)(5) at binary32 conductance G (R28), binary64."""
        return float(lib().oracle_dg(self._h, 1 if depress else 0, ctypes.c_float(G)))

    def infer(self, images: np.ndarray, T: int, seeds) -> np.ndarray:
        """NEXT-1: spike counts (n_images, n_exc) u32 with frozen weights (R21)."""
        imgs = np.ascontiguousarray(images, dtype=np.uint8).reshape(-1, self.n_in)
        sd = np.ascontiguousarray(np.asarray(seeds, dtype=np.uint64).reshape(-1))
        assert sd.size == imgs.shape[0]
        out = np.zeros((imgs.shape[0], self.n_exc), dtype=np.uint32)
        self._check(lib().oracle_infer(self._h, _ptr(imgs), imgs.shape[0], T, _ptr(sd), _ptr(out)), "oracle_infer")
        self.last_T = T
        return out

    def sparse_run(self, n_lif: int, src_off, tgt, q, images, T: int, seeds, raster: bool = False):
        """NEXT-4 (R24-R26): counts (n_trials, n_lif) u32 [, raster (n_trials, T, ceil(n_lif/32)) u32]."""
        imgs = np.ascontiguousarray(images, dtype=np.uint8).reshape(-1, self.n_in)
        so = np.ascontiguousarray(src_off, dtype=np.int32)
        tg = np.ascontiguousarray(tgt, dtype=np.uint16)
        qq = np.ascontiguousarray(q, dtype=np.uint8)
        sd = np.ascontiguousarray(np.asarray(seeds, dtype=np.uint64).reshape(-1))
        nt = imgs.shape[0]
        counts = np.zeros((nt, n_lif), dtype=np.uint32)
        r = np.zeros((nt, T, (n_lif + 31) // 32), dtype=np.uint32) if raster else None
        self._check(lib().oracle_sparse_run(self._h, self.n_in, n_lif, _ptr(so), _ptr(tg), _ptr(qq), _ptr(imgs), nt, T,
                                            _ptr(sd), _ptr(counts), _ptr(r) if raster else None), "oracle_sparse_run")
        return (counts, r) if raster else counts


def label(counts: np.ndarray, classes, n_classes: int) -> np.ndarray:
    """R22: per-neuron class label from spike counts of labelled images (-1 = never spiked)."""
    c = np.ascontiguousarray(counts, dtype=np.uint32)
    cl = np.ascontiguousarray(np.asarray(classes, dtype=np.int32).reshape(-1))
    out = np.zeros(c.shape[1], dtype=np.int32)
    rc = lib().oracle_label(_ptr(c), c.shape[0], c.shape[1], _ptr(cl), n_classes, _ptr(out))
    if rc != 0:
        raise OracleError(rc, "oracle_label")
    return out


def classify(counts: np.ndarray, labels, n_classes: int) -> np.ndarray:
    """R23: per-image predicted class by the labelled neurons' mean spike count (-1 = no vote)."""
    c = np.ascontiguousarray(counts, dtype=np.uint32)
    lb = np.ascontiguousarray(np.asarray(labels, dtype=np.int32).reshape(-1))
    out = np.zeros(c.shape[0], dtype=np.int32)
    rc = lib().oracle_classify(_ptr(c), c.shape[0], c.shape[1], _ptr(lb), n_classes, _ptr(out))
    if rc != 0:
        raise OracleError(rc, "oracle_classify")
    return out


def unpack_state(blob: np.ndarray, n_in: int, n_exc: int) -> dict:
    """Split a DESIGN.md §3.4 state blob into its fields."""
    b = np.asarray(blob, dtype=np.int32)
    hdr = b[:4]
    o = 4
    v = b[o:o + n_exc]; o += n_exc
    cnt = b[o:o + n_exc]; o += n_exc
    last_post = b[o:o + n_exc]; o += n_exc
    last_pre = b[o:o + n_in]
    vv = v.view(np.float32) if int(hdr[3]) == 0 else v
    return dict(n_in=int(hdr[0]), n_exc=int(hdr[1]), t_next=int(hdr[2]), membrane_mode=int(hdr[3]),
                v=vv.copy(), cnt=cnt.copy(), last_post=last_post.copy(), last_pre=last_pre.copy())


def unpack_bits(words: np.ndarray, n: int) -> np.ndarray:
    """(T, ceil(n/32)) u32 raster -> (T, n) bool."""
    w = np.asarray(words, dtype=np.uint32)
    if w.ndim == 1:
        w = w[None, :]
    bits = ((w[:, :, None] >> np.arange(32, dtype=np.uint32)[None, None, :]) & 1).astype(bool)
    return bits.reshape(w.shape[0], -1)[:, :n]
