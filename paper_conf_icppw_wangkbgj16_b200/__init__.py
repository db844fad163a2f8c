"""ks-b200: fused Gaussian kernel summation on NVIDIA B200 (sm_100a).

Thin ctypes binding over the C ABI in ``include/ks.h`` (``libks.so``, built
in-tree by ``paper_conf_icppw_wangkbgj16_b200.build``).  Argument
marshalling only: every step of the computation runs in the CUDA kernels of
``csrc/``.  There is no CPU fallback -- importing this package without the
built library (at first use), or calling it without an sm_100 GPU, raises.

The functions keep the C names (``ks_create``, ``ks_set_sources``, ``ks_eval``,
...).  ``KernelSum`` wraps them for torch tensors (device memory and streams
come from PyTorch; PyTorch does none of the arithmetic).

Method: Wang et al., ICPP Workshops 2016, Eq.1-2 through
Eq.3, fused as in SS III-C / Alg.2.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# KS_LIB=libks_dbg.so selects a measurement build (KS_DEBUG / KS_PROF, tools only); the
# shipped library is libks.so
LIB_PATH = os.path.join(_HERE, os.path.basename(os.environ.get("KS_LIB", "libks.so")))

KS_OK, KS_EINVAL, KS_ESTATE, KS_ENOMEM, KS_ECUDA, KS_EUNSUPPORTED = range(6)
KS_PREC_AUTO, KS_PREC_FP32, KS_PREC_3XTF32, KS_PREC_TF32, KS_PREC_3XF16 = range(5)
KS_PATH_NONE, KS_PATH_FP32, KS_PATH_TC = range(3)
PRECISIONS = {"auto": KS_PREC_AUTO, "fp32": KS_PREC_FP32, "3xtf32": KS_PREC_3XTF32, "tf32": KS_PREC_TF32,
              "3xf16": KS_PREC_3XF16}

# every symbol include/ks.h declares (checked by tests/test_abi.py)
EXPORTED = ("ks_create", "ks_destroy", "ks_set_precision", "ks_set_stream", "ks_set_sources", "ks_eval",
            "ks_set_sources_host", "ks_eval_host", "ks_reserve", "ks_get_info", "ks_timing_enable",
            "ks_timing_read", "ks_set_option", "ks_get_option", "ks_clock_read", "ks_status_str", "ks_last_error",
            "ks_version")

# tuning options (include/ks.h ks_option): variants computing the same result, none drops work
OPTIONS = {"r1_kernel": 1, "r1_epilogue": 2, "exp_poly": 3, "weighted_sum": 4, "log_weights": 5, "fold": 6,
           "aug": 7, "clamp": 8, "target_resident": 9, "stages": 10, "ar_stages": 11, "wslots": 12,
           "prep_lanes": 13, "eval_chunks": 14, "fp32_split": 15, "measure_clock": 16,
           "eval_chunk0": 17, "coop_prep": 18,
           "narrow_planes": 19}


class KsInfo(ctypes.Structure):
    _fields_ = [("path", ctypes.c_int), ("precision", ctypes.c_int), ("k_pad", ctypes.c_int),
                ("tile_t", ctypes.c_int), ("tile_s", ctypes.c_int), ("num_ctas", ctypes.c_int),
                ("stages", ctypes.c_int), ("num_sms", ctypes.c_int), ("m", ctypes.c_int64),
                ("m_pad", ctypes.c_int64), ("r", ctypes.c_int), ("launches", ctypes.c_int64),
                ("fused_launches", ctypes.c_int64), ("c_log2", ctypes.c_double), ("kernel", ctypes.c_int),
                ("exp_poly", ctypes.c_int), ("r1_epilogue", ctypes.c_int)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class KsError(RuntimeError):
    def __init__(self, status, where, detail):
        self.status = status
        super().__init__(f"{where}: {status_str(status)}: {detail}")


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(
            f"libks.so not found at {LIB_PATH}: build it with "
            "`python -m paper_conf_icppw_wangkbgj16_b200.build` (no CPU fallback exists)")
    lib = ctypes.CDLL(LIB_PATH)
    P, I, L, F, D = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_float, ctypes.c_double
    sig = {
        "ks_create": ([I, F, ctypes.POINTER(P)], I),
        "ks_destroy": ([P], I),
        "ks_set_precision": ([P, I], I),
        "ks_set_stream": ([P, P], I),
        "ks_set_sources": ([P, P, P, L, I], I),
        "ks_eval": ([P, P, L, P], I),
        "ks_set_sources_host": ([P, P, P, L, I], I),
        "ks_eval_host": ([P, P, L, P], I),
        "ks_reserve": ([P, L], I),
        "ks_get_info": ([P, ctypes.POINTER(KsInfo)], I),
        "ks_timing_enable": ([P, I], I),
        "ks_timing_read": ([P, ctypes.POINTER(D), ctypes.POINTER(L), I], I),
        "ks_set_option": ([P, I, I], I),
        "ks_get_option": ([P, I, ctypes.POINTER(I)], I),
        "ks_clock_read": ([P, ctypes.POINTER(D), ctypes.POINTER(I)], I),
        "ks_status_str": ([I], ctypes.c_char_p),
        "ks_last_error": ([], ctypes.c_char_p),
        "ks_version": ([], ctypes.c_char_p),
    }
    for name, (args, res) in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = res
    return lib


class _Lazy:
    """Loads libks.so at first use and raises ImportError if it is missing
    (lazy only so that ``paper_conf_icppw_wangkbgj16_b200.build`` can be
    imported to build it)."""

    _lib = None

    def __getattr__(self, name):
        if _Lazy._lib is None:
            _Lazy._lib = _load()
        return getattr(_Lazy._lib, name)


_lib = _Lazy()


def load():
    """Force-load libks.so now (raises ImportError if it has not been built)."""
    _lib.ks_version
    return _Lazy._lib


def status_str(s: int) -> str:
    return _lib.ks_status_str(int(s)).decode()


def last_error() -> str:
    return _lib.ks_last_error().decode()


def version() -> str:
    return _lib.ks_version().decode()


def _check(status, where):
    if status != KS_OK:
        raise KsError(status, where, last_error())


# ---------------------------------------------------------------- C names
def ks_create(K: int, h: float) -> int:
    h_out = ctypes.c_void_p()
    _check(_lib.ks_create(int(K), float(h), ctypes.byref(h_out)), "ks_create")
    return h_out.value


def ks_destroy(ctx) -> None:
    _check(_lib.ks_destroy(ctx), "ks_destroy")


def ks_set_precision(ctx, p) -> None:
    if isinstance(p, str):
        p = PRECISIONS[p.lower()]
    _check(_lib.ks_set_precision(ctx, int(p)), "ks_set_precision")


def ks_set_stream(ctx, stream_ptr: int) -> None:
    _check(_lib.ks_set_stream(ctx, ctypes.c_void_p(int(stream_ptr))), "ks_set_stream")


def ks_set_sources(ctx, alpha_ptr: int, W_ptr: int, M: int, R: int) -> None:
    _check(_lib.ks_set_sources(ctx, alpha_ptr, W_ptr, int(M), int(R)), "ks_set_sources")


def ks_eval(ctx, beta_ptr: int, N: int, V_ptr: int) -> None:
    _check(_lib.ks_eval(ctx, beta_ptr, int(N), V_ptr), "ks_eval")


def ks_set_sources_host(ctx, alpha_ptr: int, W_ptr: int, M: int, R: int) -> None:
    _check(_lib.ks_set_sources_host(ctx, alpha_ptr, W_ptr, int(M), int(R)), "ks_set_sources_host")


def ks_eval_host(ctx, beta_ptr: int, N: int, V_ptr: int) -> None:
    _check(_lib.ks_eval_host(ctx, beta_ptr, int(N), V_ptr), "ks_eval_host")


def ks_reserve(ctx, N_max: int) -> None:
    _check(_lib.ks_reserve(ctx, int(N_max)), "ks_reserve")


def ks_get_info(ctx) -> dict:
    info = KsInfo()
    _check(_lib.ks_get_info(ctx, ctypes.byref(info)), "ks_get_info")
    return info.as_dict()


def ks_set_option(ctx, opt, value: int) -> None:
    if isinstance(opt, str):
        opt = OPTIONS[opt]
    _check(_lib.ks_set_option(ctx, int(opt), int(value)), "ks_set_option")


def ks_get_option(ctx, opt) -> int:
    if isinstance(opt, str):
        opt = OPTIONS[opt]
    v = ctypes.c_int()
    _check(_lib.ks_get_option(ctx, int(opt), ctypes.byref(v)), "ks_get_option")
    return v.value


def ks_clock_read(ctx):
    """(effective SM GHz, CTAs) of the last fused launch measured with option measure_clock=1."""
    g = ctypes.c_double()
    n = ctypes.c_int()
    _check(_lib.ks_clock_read(ctx, ctypes.byref(g), ctypes.byref(n)), "ks_clock_read")
    return g.value, n.value


def ks_timing_enable(ctx, on: bool) -> None:
    _check(_lib.ks_timing_enable(ctx, 1 if on else 0), "ks_timing_enable")


def ks_timing_read(ctx, reset: bool = True):
    ms = ctypes.c_double()
    n = ctypes.c_int64()
    _check(_lib.ks_timing_read(ctx, ctypes.byref(ms), ctypes.byref(n), 1 if reset else 0), "ks_timing_read")
    return ms.value, n.value


# ---------------------------------------------------------------- torch wrapper
class KernelSum:
    """One context: ``KernelSum(K, h)``, ``set_sources(alpha, W)``, ``eval(beta) -> V``.

    Tensors: FP32, contiguous, on the context's CUDA device (``eval`` allocates
    V unless ``out`` is given).  Work is ordered on the current torch stream
    at call time.  ``set_sources_host`` / ``eval_host`` take numpy arrays or
    CPU tensors and include the host<->device copies.
    """

    def __init__(self, K: int, h: float, precision: str = "auto", options: dict | None = None):
        import torch
        load()
        self._torch = torch
        if not torch.cuda.is_available():
            raise RuntimeError("KernelSum needs a CUDA device (no CPU fallback)")
        self.K = int(K)
        self.h = float(h)
        self.device = torch.cuda.current_device()
        self.ctx = ks_create(self.K, self.h)
        ks_set_precision(self.ctx, precision)
        for k, v in (options or {}).items():
            ks_set_option(self.ctx, k, v)
        self.R = 1
        self.M = 0

    def set_option(self, name, value: int):
        ks_set_option(self.ctx, name, value)

    def get_option(self, name) -> int:
        return ks_get_option(self.ctx, name)

    def close(self):
        if getattr(self, "ctx", None):
            ks_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def _stream(self):
        ks_set_stream(self.ctx, self._torch.cuda.current_stream().cuda_stream)

    def _dev(self, t, name, shape1, rows=None):
        torch = self._torch
        if not isinstance(t, torch.Tensor) or not t.is_cuda or t.dtype != torch.float32:
            raise TypeError(f"{name} must be a CUDA float32 tensor")
        if t.device.index != self.device:
            raise ValueError(f"{name} is on cuda:{t.device.index}, the context on cuda:{self.device}")
        if not t.is_contiguous():
            raise ValueError(f"{name} must be contiguous")
        if t.dim() != 2 or t.shape[1] != shape1 or (rows is not None and t.shape[0] != rows):
            want = f"[{'n' if rows is None else rows}, {shape1}]"
            raise ValueError(f"{name} must be {want}, got {tuple(t.shape)}")
        return t

    @staticmethod
    def _host(x, name, shape1, rows=None):
        import numpy as np
        a = np.ascontiguousarray(x, dtype=np.float32)
        if a.ndim != 2 or a.shape[1] != shape1 or (rows is not None and a.shape[0] != rows):
            want = f"[{'n' if rows is None else rows}, {shape1}]"
            raise ValueError(f"{name} must be {want}, got {tuple(a.shape)}")
        return a

    def set_sources(self, alpha, W):
        if W.dim() == 1:
            W = W.reshape(-1, 1)
        alpha = self._dev(alpha, "alpha", self.K)
        W = self._dev(W, "W", W.shape[1], rows=alpha.shape[0])
        self._stream()
        ks_set_sources(self.ctx, alpha.data_ptr(), W.data_ptr(), alpha.shape[0], W.shape[1])
        self.M, self.R = alpha.shape[0], W.shape[1]
        self._keep = (alpha, W)  # stream-ordered: keep alive until the next set

    def eval(self, beta, out=None):
        beta = self._dev(beta, "beta", self.K)
        N = beta.shape[0]
        if out is None:
            out = self._torch.empty((N, self.R), dtype=self._torch.float32, device=beta.device)
        else:
            out = self._dev(out, "out", self.R, rows=N)
        self._stream()
        ks_eval(self.ctx, beta.data_ptr(), N, out.data_ptr())
        return out

    def set_sources_host(self, alpha, W):
        import numpy as np
        a = self._host(alpha, "alpha", self.K)
        w = np.asarray(W, dtype=np.float32)
        if w.ndim == 1:
            w = w[:, None]
        w = self._host(w, "W", w.shape[1] if w.ndim == 2 else -1, rows=a.shape[0])
        self._stream()
        ks_set_sources_host(self.ctx, a.ctypes.data, w.ctypes.data, a.shape[0], w.shape[1])
        self.M, self.R = a.shape[0], w.shape[1]

    def eval_host(self, beta, out=None):
        import numpy as np
        b = self._host(beta, "beta", self.K)
        if out is None:
            out = np.empty((b.shape[0], self.R), dtype=np.float32)
        elif (not isinstance(out, np.ndarray) or out.dtype != np.float32 or out.shape != (b.shape[0], self.R)
              or not out.flags["C_CONTIGUOUS"]):
            raise ValueError(f"out must be a C-contiguous float32 array of shape {(b.shape[0], self.R)}")
        self._stream()
        ks_eval_host(self.ctx, b.ctypes.data, b.shape[0], out.ctypes.data)
        return out

    def info(self) -> dict:
        return ks_get_info(self.ctx)
