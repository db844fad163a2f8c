"""CPU oracle for fused Gaussian kernel summation -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product path (``paper_conf_icppw_wangkbgj16_b200``) never imports it and
shares no code with it.

``oracle_eval`` is the plain FP64 definition of Eq.1-2 (PAPER.md P:L24-38,
SS I) written out as a double loop in ``oracle.c``; see that file's header for
the readings taken (SS3) and ``tests/test_oracle_pins.py`` for what
pins it.

Parity: pinned (closed forms, brute-force hand cases, invariants, an
independent numpy Alg.1 formulation, a separable closed form at the headline
shape).  No function here is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so with gcc -O2 -fopenmp (no -ffast-math:
    the oracle must keep IEEE semantics)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(
            ["gcc", "-O2", "-fno-fast-math", "-ffp-contract=off", "-fopenmp", "-fPIC",
             "-shared", "-std=c11", _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _bind(path):
    lib = ctypes.CDLL(path)
    lib.oracle_eval.restype = ctypes.c_int
    lib.oracle_eval.argtypes = [
        ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int,
        ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_double,
        ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p]
    lib.oracle_num_threads.restype = ctypes.c_int
    lib.oracle_set_num_threads.argtypes = [ctypes.c_int]
    return lib


def _load():
    global _lib
    if _lib is None:
        build()
        _lib = _bind(_LIB)
    return _lib


def num_threads() -> int:
    return int(_load().oracle_num_threads())


def set_num_threads(n: int) -> None:
    _load().oracle_set_num_threads(int(n))


def oracle_eval(alpha, W, beta, h, J=None, want_S=False, _lib_override=None):
    """V[t, r] = sum_i exp(-||alpha_i - beta_{J[t]}||^2 / (2 h^2)) W[i, r]  (Eq.1-2).

    alpha [M, K] f32, W [M] or [M, R] f32, beta [N, K] f32, h float (widened
    from the FP32 value the GPU receives).  J: optional int64 target subset.
    Returns V [nJ, R] f64 (and S = sum_i K |W| if want_S).
    """
    lib = _lib_override if _lib_override is not None else _load()
    alpha = np.ascontiguousarray(alpha, dtype=np.float32)
    beta = np.ascontiguousarray(beta, dtype=np.float32)
    W = np.asarray(W, dtype=np.float32)
    if W.ndim == 1:
        W = W[:, None]
    W = np.ascontiguousarray(W)
    M, K = alpha.shape
    N = beta.shape[0]
    if beta.shape[1] != K:
        raise ValueError("alpha and beta must have the same K")
    R = W.shape[1]
    if W.shape[0] != M:
        raise ValueError("W rows must equal M")
    if J is not None:
        J = np.ascontiguousarray(J, dtype=np.int64)
        nJ = J.shape[0]
    else:
        nJ = N
    V = np.zeros((nJ, R), dtype=np.float64)
    S = np.zeros((nJ, R), dtype=np.float64) if want_S else None
    rc = lib.oracle_eval(
        alpha.ctypes.data if M else None, W.ctypes.data if M else None, M, R,
        beta.ctypes.data if N else None, N, K, float(h),
        J.ctypes.data if J is not None and nJ else None, nJ,
        V.ctypes.data if nJ else None, S.ctypes.data if (S is not None and nJ) else None)
    if rc != 0:
        raise ValueError(f"oracle_eval rejected arguments (rc={rc})")
    return (V, S) if want_S else V


class Variant:
    """An oracle built from another source text (used only by the mutation
    self-test, tests/test_oracle_mutants.py, to show the pins catch bugs)."""

    def __init__(self, path):
        self._lib = _bind(path)

    def oracle_eval(self, *a, **kw):
        return oracle_eval(*a, _lib_override=self._lib, **kw)

    def num_threads(self):
        return int(self._lib.oracle_num_threads())

    def set_num_threads(self, n):
        self._lib.oracle_set_num_threads(int(n))
