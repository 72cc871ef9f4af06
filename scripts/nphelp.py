"""numpy one-liners the measurement scripts use for spot checks (the oracle package is
test infrastructure: tests/, smoke() and bench.py's cpu_baseline leg only)."""
import numpy as np


def scatter_np(p, a):
    b = np.empty_like(a)
    b[p] = a
    return b


def inverse_np(p):
    q = np.empty_like(p)
    q[p] = np.arange(p.size, dtype=p.dtype)
    return q
