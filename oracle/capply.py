"""ctypes loader for oracle/c/apply_ref.c. ORACLE — test infrastructure only.

Builds the plain C definition loop on first use if the shared
object is missing. Used only to time the oracle on the host cores.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(_HERE, "c", "apply_ref.c")
LIB = os.path.join(_HERE, "c", "liboracle_apply.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", SRC, "-o", LIB])
    return LIB


def _load():
    global _lib
    if _lib is None:
        build()
        _lib = ctypes.CDLL(LIB)
        for name in ("oracle_apply_u32", "oracle_apply_u64"):
            f = getattr(_lib, name)
            f.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64]
            f.restype = None
        _lib.oracle_threads.restype = ctypes.c_int
    return _lib


def threads() -> int:
    return int(_load().oracle_threads())


def apply_c(p: np.ndarray, a: np.ndarray, out: np.ndarray | None = None) -> np.ndarray:
    """b[p[i]] = a[i] via the plain C loop. p int32, a uint32/uint64 (raw words)."""
    lib = _load()
    p = np.ascontiguousarray(p, dtype=np.int32)
    a = np.ascontiguousarray(a)
    if out is None:
        out = np.empty_like(a)
    fn = lib.oracle_apply_u32 if a.dtype.itemsize == 4 else lib.oracle_apply_u64
    fn(p.ctypes.data, a.ctypes.data, out.ctypes.data, a.size)
    return out
