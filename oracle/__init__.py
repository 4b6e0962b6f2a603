"""ORACLE package — TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct CPU references for the PolyHankel hot path
(§2.2 Eq. 4-12, §3.2).  Only tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / --impl reference legs may import this package.  The
product path (paper_conf_cgo_xuzc025_b200) never imports it and shares no code
with it; the only module both sides use is synth/ (seeded input generators,
no method arithmetic).

  conv2d(x, w, stride, padding)  O1: fp64 direct convolution, plain C
                                 (conv_ref.c), the gate oracle.
  poly_ref                       O2: the method step by step (numpy), degree
                                 maps, packing/rounding references.

Parity status: every function is pinned by tests/test_oracle_pins.py against
paper-printed values, closed forms, library special cases or invariants
(DESIGN.md §Oracle lists each pin).  No function is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from . import poly_ref  # noqa: F401

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "conv_ref.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile conv_ref.c with gcc -O2 -fopenmp (no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c99",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        dp = ctypes.POINTER(ctypes.c_double)
        lib.oracle_conv2d_f64.argtypes = [dp, dp, dp] + [ctypes.c_int] * 12
        lib.oracle_conv2d_f64.restype = ctypes.c_int
        lib.oracle_output_dims.argtypes = [ctypes.c_int] * 8 + [ctypes.POINTER(ctypes.c_int)] * 2
        lib.oracle_output_dims.restype = ctypes.c_int
        lib.oracle_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def output_dims(H, W, R, S, stride=(1, 1), padding=(0, 0)):
    P, Q = ctypes.c_int(), ctypes.c_int()
    rc = _load().oracle_output_dims(H, W, R, S, stride[0], stride[1], padding[0], padding[1],
                                    ctypes.byref(P), ctypes.byref(Q))
    if rc:
        raise ValueError("bad convolution parameters")
    return P.value, Q.value


def conv2d(x, w, stride=(1, 1), padding=(0, 0), threads: int = 0) -> np.ndarray:
    """O1: y = conv(x, w) in fp64.  x[N][C][H][W], w[K][C][R][S] (any real
    dtype; fp32 values widen exactly).  threads=0 -> OpenMP default."""
    x = np.ascontiguousarray(x, dtype=np.float64)
    w = np.ascontiguousarray(w, dtype=np.float64)
    N, C, H, W = x.shape
    K, C2, R, S = w.shape
    if C != C2:
        raise ValueError("channel mismatch")
    P, Q = output_dims(H, W, R, S, stride, padding)
    y = np.empty((N, K, P, Q), dtype=np.float64)
    dp = ctypes.POINTER(ctypes.c_double)
    rc = _load().oracle_conv2d_f64(x.ctypes.data_as(dp), w.ctypes.data_as(dp), y.ctypes.data_as(dp),
                                   N, C, H, W, K, R, S, stride[0], stride[1], padding[0], padding[1],
                                   int(threads))
    if rc:
        raise ValueError("bad convolution parameters")
    return y


def max_threads() -> int:
    return int(_load().oracle_max_threads())
