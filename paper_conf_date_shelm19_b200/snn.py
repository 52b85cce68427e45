"""Thin ctypes binding of include/snn.h (libsnn_b200.so).  Argument marshalling only: every step
of the simulate-and-learn path runs in the library's CUDA kernels.  There is no CPU fallback:
if the in-tree extension is missing this module raises on import of the library."""
from __future__ import annotations

import ctypes
import os
from typing import Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SNN_LIB_PATH") or os.path.join(_HERE, "libsnn_b200.so")   # override: experiments only

SNN_OK, SNN_EINVAL, SNN_ENOMEM, SNN_ECUDA, SNN_ENCCL, SNN_ESIZE, SNN_ECOOP = 0, -1, -2, -3, -4, -5, -6
SNN_RASTER_INPUT, SNN_KEEP_STATE, SNN_RECORD_INPUT, SNN_ASYNC, SNN_FLOOR_PROBE = 1, 2, 4, 8, 16
PRESETS = {"2b": 0, "4b": 1, "8b": 2, "16b": 3, "hf": 4}

# Every function declared in include/snn.h (checked by tests/test_abi.py).
EXPORTS = [
    "snn_params_preset", "snn_create", "snn_destroy", "snn_set_stream", "snn_synchronize",
    "snn_present", "snn_present_batch", "snn_present_ex", "snn_present_raster", "snn_present_many", "snn_infer_many",
    "snn_get_weights", "snn_set_weights", "snn_get_spikes", "snn_get_input_raster",
    "snn_state_bytes", "snn_get_state", "snn_set_state", "snn_get_stats", "snn_reset_stats",
    "snn_get_info", "snn_set_trace", "snn_get_trace", "snn_set_profile", "snn_get_profile", "snn_last_error",
    "snn_create_shard", "snn_shard_ipc_handle", "snn_shard_connect", "snn_shard_link",
    "snn_infer", "snn_get_infer_stats", "snn_label", "snn_classify",
    "snn_sparse_run", "snn_get_sparse_stats",
]
SNN_IPC_HANDLE_BYTES = 64
NINFO = 18


class SnnParams(ctypes.Structure):
    """snn_params (include/snn.h)."""
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
        ("cluster_size", ctypes.c_int32), ("engine", ctypes.c_int32),
    ]

    def as_dict(self) -> dict:
        return {name: getattr(self, name) for name, _ in self._fields_}


_lib = None


def lib():
    """Load the in-tree CUDA library (raises if it was not built: no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"CUDA extension not built: {LIB_PATH} (run __graft_entry__.build())")
        L = ctypes.CDLL(LIB_PATH)
        vp, i32, u64, sz = ctypes.c_void_p, ctypes.c_int, ctypes.c_uint64, ctypes.c_size_t
        pp = ctypes.POINTER(SnnParams)
        sig = {
            "snn_params_preset": ([pp, i32], i32),
            "snn_create": ([i32, i32, i32, pp, ctypes.POINTER(vp)], i32),
            "snn_destroy": ([vp], i32),
            "snn_set_stream": ([vp, vp], i32),
            "snn_synchronize": ([vp], i32),
            "snn_present": ([vp, vp, i32, u64], i32),
            "snn_present_batch": ([vp, vp, i32, i32, vp, vp, i32], i32),
            "snn_present_ex": ([vp, vp, i32, u64, i32, i32], i32),
            "snn_present_raster": ([vp, vp, i32, u64], i32),
            "snn_present_many": ([vp, i32, vp, i32, i32, vp], i32),
            "snn_infer_many": ([vp, i32, vp, i32, i32, vp, vp], i32),
            "snn_get_weights": ([vp, vp, sz], i32),
            "snn_set_weights": ([vp, vp, sz], i32),
            "snn_get_spikes": ([vp, vp, sz], i32),
            "snn_get_input_raster": ([vp, vp, sz], i32),
            "snn_state_bytes": ([vp], sz),
            "snn_get_state": ([vp, vp, sz], i32),
            "snn_set_state": ([vp, vp, sz], i32),
            "snn_get_stats": ([vp, vp], i32),
            "snn_reset_stats": ([vp], i32),
            "snn_get_info": ([vp, vp], i32),
            "snn_set_trace": ([vp, i32], i32),
            "snn_get_trace": ([vp, vp, sz], i32),
            "snn_set_profile": ([vp, i32], i32),
            "snn_get_profile": ([vp, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_int64)], i32),
            "snn_last_error": ([], ctypes.c_char_p),
            "snn_create_shard": ([i32, i32, i32, pp, i32, i32, ctypes.POINTER(vp)], i32),
            "snn_shard_ipc_handle": ([vp, vp, sz], i32),
            "snn_shard_connect": ([vp, vp, sz], i32),
            "snn_shard_link": ([vp, i32], i32),
            "snn_infer": ([vp, vp, i32, i32, vp, vp, i32], i32),
            "snn_get_infer_stats": ([vp, vp], i32),
            "snn_label": ([vp, vp, i32, vp, i32, vp], i32),
            "snn_classify": ([vp, vp, i32, vp, i32, vp], i32),
            "snn_sparse_run": ([vp, i32, vp, vp, vp, vp, i32, i32, vp, vp, vp, i32], i32),
            "snn_get_sparse_stats": ([vp, vp], i32),
        }
        for name, (args, res) in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = res
        _lib = L
    return _lib


class SnnError(RuntimeError):
    def __init__(self, rc: int, what: str):
        msg = lib().snn_last_error().decode(errors="replace")
        super().__init__(f"{what} failed rc={rc}: {msg}")
        self.rc = rc


def _check(rc: int, what: str):
    if rc != SNN_OK:
        raise SnnError(rc, what)


def preset(name: str = "8b", **overrides) -> SnnParams:
    p = SnnParams()
    _check(lib().snn_params_preset(ctypes.byref(p), PRESETS[name]), "snn_params_preset")
    for k, v in overrides.items():
        if not hasattr(p, k):
            raise KeyError(k)
        setattr(p, k, v)
    return p


def params_from_dict(d: dict, **overrides) -> SnnParams:
    """Parameter block from a dict of DESIGN.md §3.1 fields (`engine` defaults to event-driven)."""
    p = SnnParams()
    for name, _ in SnnParams._fields_:
        if name == "engine":
            p.engine = int(d.get("engine", 0))
        else:
            setattr(p, name, d[name])
    for k, v in overrides.items():
        setattr(p, k, v)
    return p


def _ptr(x) -> ctypes.c_void_p:
    """Host numpy array or torch tensor (host or CUDA) -> raw pointer."""
    if x is None:
        return ctypes.c_void_p(0)
    if isinstance(x, np.ndarray):
        assert x.flags["C_CONTIGUOUS"]
        return ctypes.c_void_p(x.ctypes.data)
    if hasattr(x, "data_ptr"):
        assert x.is_contiguous()
        return ctypes.c_void_p(x.data_ptr())
    raise TypeError(type(x))


class Network:
    """One snn_handle: n_in -> n_exc network with `bits`-bit conductance codes on the GPU."""

    def __init__(self, n_in: int, n_exc: int, bits: int, params: Optional[SnnParams] = None,
                 shard: Optional[tuple] = None, **overrides):
        """shard=(rank, world): this object is shard `rank` of an n_exc-column network split over
        `world` ranks (include/snn.h snn_create_shard); self.n_exc becomes the shard's own columns."""
        self.n_in, self.n_exc, self.bits = n_in, n_exc, bits
        self.params = params if params is not None else preset({2: "2b", 4: "4b", 8: "8b", 16: "16b", 32: "16b"}[bits])
        for k, v in overrides.items():
            setattr(self.params, k, v)
        self._h = ctypes.c_void_p()
        if shard is None:
            _check(lib().snn_create(n_in, n_exc, bits, ctypes.byref(self.params), ctypes.byref(self._h)), "snn_create")
            self.col_base, self.n_exc_total = 0, n_exc
        else:
            rank, world = shard
            _check(lib().snn_create_shard(n_in, n_exc, bits, ctypes.byref(self.params), rank, world,
                                          ctypes.byref(self._h)), "snn_create_shard")
            inf = self.info()
            self.col_base, self.n_exc_total = inf["col_base"], inf["n_exc_total"]
            self.n_exc = (min(self.n_exc_total, 32 * (((rank + 1) * ((n_exc + 31) // 32)) // world))
                          - self.col_base)
        self.last_T = 0

    @property
    def handle(self) -> ctypes.c_void_p:
        return self._h

    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            lib().snn_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def info(self) -> dict:
        a = (ctypes.c_int64 * NINFO)()
        _check(lib().snn_get_info(self._h, a), "snn_get_info")
        keys = ["cluster_size", "threads", "smem_bytes", "words_per_row", "q_max", "L_pot", "L_dep", "launches",
                "engine", "cols_per_thread", "row_window", "log_depth", "col_base", "n_exc_total", "world", "shard",
                "lean", "smem_lean"]
        return dict(zip(keys, [int(x) for x in a]))

    def set_stream(self, stream_ptr: int):
        _check(lib().snn_set_stream(self._h, ctypes.c_void_p(stream_ptr)), "snn_set_stream")

    def synchronize(self):
        _check(lib().snn_synchronize(self._h), "snn_synchronize")

    def present(self, image, T: int, seed: int):
        _check(lib().snn_present(self._h, _ptr(image), T, seed), "snn_present")
        self.last_T = T

    def present_ex(self, inp, T: int, seed: int, flags: int = 0, t0: int = 0):
        _check(lib().snn_present_ex(self._h, _ptr(inp), T, seed, flags, t0), "snn_present_ex")
        self.last_T = T

    def present_raster(self, raster, T: int, seed: int, keep_state: bool = False, t0: int = 0):
        flags = SNN_RASTER_INPUT | (SNN_KEEP_STATE if keep_state else 0)
        self.present_ex(raster, T, seed, flags, t0)

    def present_batch(self, images, T: int, seeds, spike_counts=None, flags: int = 0):
        n = int(images.shape[0])
        _check(lib().snn_present_batch(self._h, _ptr(images), n, T, _ptr(seeds), _ptr(spike_counts), flags),
               "snn_present_batch")
        self.last_T = T

    @property
    def code_dtype(self):
        """uint8 codes (<= 8 bits), uint16 codes (16 bits), binary32 conductance (32 bits, R28)"""
        return np.float32 if self.bits == 32 else (np.uint16 if self.bits > 8 else np.uint8)

    def weights(self) -> np.ndarray:
        out = np.empty((self.n_in, self.n_exc), dtype=self.code_dtype)
        _check(lib().snn_get_weights(self._h, _ptr(out), out.nbytes), "snn_get_weights")
        return out

    def set_weights(self, codes: np.ndarray):
        c = np.ascontiguousarray(codes, dtype=self.code_dtype).reshape(self.n_in, self.n_exc)
        _check(lib().snn_set_weights(self._h, _ptr(c), c.nbytes), "snn_set_weights")

    def spikes(self) -> np.ndarray:
        we = (self.n_exc + 31) // 32
        out = np.zeros((self.last_T, we), dtype=np.uint32)
        _check(lib().snn_get_spikes(self._h, _ptr(out), out.size), "snn_get_spikes")
        return out

    def input_raster(self) -> np.ndarray:
        wi = (self.n_in + 31) // 32
        out = np.zeros((self.last_T, wi), dtype=np.uint32)
        _check(lib().snn_get_input_raster(self._h, _ptr(out), out.size), "snn_get_input_raster")
        return out

    def state(self) -> np.ndarray:
        n = int(lib().snn_state_bytes(self._h))
        out = np.zeros(n // 4, dtype=np.int32)
        _check(lib().snn_get_state(self._h, _ptr(out), out.nbytes), "snn_get_state")
        return out

    def set_state(self, blob: np.ndarray):
        b = np.ascontiguousarray(blob, dtype=np.int32)
        _check(lib().snn_set_state(self._h, _ptr(b), b.nbytes), "snn_set_state")

    def stats(self) -> np.ndarray:
        out = np.zeros(16, dtype=np.uint64)
        _check(lib().snn_get_stats(self._h, _ptr(out)), "snn_get_stats")
        return out

    def set_trace(self, max_epochs: int):
        _check(lib().snn_set_trace(self._h, max_epochs), "snn_set_trace")
        self._trace_epochs = max_epochs

    def trace(self) -> np.ndarray:
        """(cluster_size, max_epochs, 8) u64 per-epoch records (include/snn.h snn_set_trace)."""
        cs = self.info()["cluster_size"]
        out = np.zeros((cs, self._trace_epochs, 8), dtype=np.uint64)
        _check(lib().snn_get_trace(self._h, _ptr(out), out.size), "snn_get_trace")
        return out

    def reset_stats(self):
        _check(lib().snn_reset_stats(self._h), "snn_reset_stats")

    def set_profile(self, on: bool = True):
        """CUDA events around every presentation kernel on the handle's stream (include/snn.h)."""
        _check(lib().snn_set_profile(self._h, 1 if on else 0), "snn_set_profile")

    def profile(self):
        """-> (summed presentation-kernel milliseconds, kernels) since the last call; resets."""
        ms, n = ctypes.c_double(0.0), ctypes.c_int64(0)
        _check(lib().snn_get_profile(self._h, ctypes.byref(ms), ctypes.byref(n)), "snn_get_profile")
        return ms.value, n.value

    # ---- NEXT-1: inference with frozen weights, labelling, vote (include/snn.h)
    def infer(self, images, T: int, seeds, counts=None, flags: int = 0):
        """Spike counts (n_images, n_exc) u32 of each image presented with frozen weights.  images/seeds/
        counts: numpy (host) or torch CUDA tensors; counts is allocated on the host if not given."""
        n = int(images.shape[0])
        if counts is None:
            counts = np.zeros((n, self.n_exc), dtype=np.uint32)
        _check(lib().snn_infer(self._h, _ptr(images), n, T, _ptr(seeds), _ptr(counts), flags), "snn_infer")
        return counts

    def infer_stats(self) -> np.ndarray:
        """[active input rows, post spikes, LIF column-steps run] summed over every inference call."""
        out = np.zeros(3, dtype=np.uint64)
        _check(lib().snn_get_infer_stats(self._h, _ptr(out)), "snn_get_infer_stats")
        return out

    def label(self, counts, classes, n_classes: int, labels=None):
        n = int(counts.shape[0])
        if labels is None:
            labels = np.zeros(self.n_exc, dtype=np.int32)
        _check(lib().snn_label(self._h, _ptr(counts), n, _ptr(classes), n_classes, _ptr(labels)), "snn_label")
        return labels

    def classify(self, counts, labels, n_classes: int, pred=None):
        n = int(counts.shape[0])
        if pred is None:
            pred = np.zeros(n, dtype=np.int32)
        _check(lib().snn_classify(self._h, _ptr(counts), n, _ptr(labels), n_classes, _ptr(pred)), "snn_classify")
        return pred

    # ---- NEXT-4: the Fig. 4 sparse workload (include/snn.h snn_sparse_run)
    def sparse_run(self, n_lif: int, src_off, tgt, q, images, T: int, seeds, counts=None, raster=None,
                   flags: int = 0):
        """Spike counts (n_trials, n_lif) u32 of the sparse recurrent network (this handle's parameters);
        raster: optional (n_trials, T, ceil(n_lif/32)) u32 output buffer."""
        n = int(images.shape[0])
        if counts is None:
            counts = np.zeros((n, n_lif), dtype=np.uint32)
        _check(lib().snn_sparse_run(self._h, n_lif, _ptr(src_off), _ptr(tgt), _ptr(q), _ptr(images), n, T,
                                    _ptr(seeds), _ptr(counts), _ptr(raster), flags), "snn_sparse_run")
        return counts

    def sparse_stats(self) -> np.ndarray:
        out = np.zeros(2, dtype=np.uint64)
        _check(lib().snn_get_sparse_stats(self._h, _ptr(out)), "snn_get_sparse_stats")
        return out

    # ---- column sharding (include/snn.h)
    def ipc_handle(self) -> bytes:
        buf = ctypes.create_string_buffer(SNN_IPC_HANDLE_BYTES)
        _check(lib().snn_shard_ipc_handle(self._h, buf, SNN_IPC_HANDLE_BYTES), "snn_shard_ipc_handle")
        return buf.raw

    def connect(self, handles: Sequence[bytes]):
        """Open every rank's mailbox (handles in rank order, this rank's own included)."""
        blob = b"".join(handles)
        _check(lib().snn_shard_connect(self._h, ctypes.c_char_p(blob), len(blob)), "snn_shard_connect")


def link_shards(shards: Sequence[Network]):
    """Single process: link shards 0..world-1 of one network (include/snn.h snn_shard_link)."""
    hs = (ctypes.c_void_p * len(shards))(*[x.handle.value for x in shards])
    _check(lib().snn_shard_link(hs, len(shards)), "snn_shard_link")


def infer_many(nets: Sequence[Network], images: Sequence, T: int, seeds: Sequence):
    """Inference with frozen weights for several per-step-engine networks (or the shards of one) in one launch;
    returns one (n_images, n_exc) u32 count array per network (include/snn.h snn_infer_many)."""
    n = len(nets)
    n_images = int(images[0].shape[0])
    outs = [np.zeros((n_images, x.n_exc), dtype=np.uint32) for x in nets]
    hs = (ctypes.c_void_p * n)(*[x.handle.value for x in nets])
    imgs = (ctypes.c_void_p * n)(*[_ptr(a).value for a in images])
    sds = (ctypes.c_void_p * n)(*[_ptr(s).value for s in seeds])
    cts = (ctypes.c_void_p * n)(*[_ptr(c).value for c in outs])
    _check(lib().snn_infer_many(hs, n, imgs, n_images, T, sds, cts), "snn_infer_many")
    return outs


def present_many(nets: Sequence[Network], images: Sequence, T: int, seeds: Sequence):
    """Ensemble: every network presents its own image batch, all in one kernel launch."""
    n = len(nets)
    hs = (ctypes.c_void_p * n)(*[x.handle.value for x in nets])
    imgs = (ctypes.c_void_p * n)(*[_ptr(a).value for a in images])
    sds = (ctypes.c_void_p * n)(*[_ptr(s).value for s in seeds])
    n_images = int(images[0].shape[0])
    _check(lib().snn_present_many(hs, n, imgs, n_images, T, sds), "snn_present_many")
    for x in nets:
        x.last_T = T
