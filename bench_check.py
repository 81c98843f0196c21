"""Bench-side sanity checks of the device results (sampled), written out here with NumPy.

The oracle (`oracle/`) is test infrastructure that only `tests/`, `__graft_entry__.smoke()` and
bench.py's cpu_baseline / --impl reference legs may run; the bench lines still report a sampled
correctness check of what they timed, so these few reference computations are restated here
(fp64, same definitions as SURVEY §8(c) O1), together with the two scheduling metrics the queue
bench reports (ANTT and STP, Eyerman [14]: P:293).
"""
from __future__ import annotations

import numpy as np


def saxpy_i32(a: int, x: np.ndarray, y: np.ndarray) -> np.ndarray:
    """y' = a*x + y modulo 2^32 (two's complement)."""
    r = (np.int64(a) * x.astype(np.int64) + y.astype(np.int64)) & 0xFFFFFFFF
    return r.astype(np.uint32).view(np.int32)


def spmv_row(col: np.ndarray, val: np.ndarray, x: np.ndarray):
    """One CSR row in fp64: (sum_p val[p] x[col[p]], sum_p |val[p] x[col[p]]|)."""
    p = val.astype(np.float64) * x[col].astype(np.float64)
    return float(p.sum()), float(np.abs(p).sum())


def stencil5_f32(a: np.ndarray):
    """5-point sweep in fp64 (0.5 c + 0.125 (n + s + w + e) inside, boundary copied) and the
    per-cell sum of |terms| (cancellation-safe denominator)."""
    a = a.astype(np.float64)
    out = a.copy()
    den = np.abs(a).copy()
    c, n, s, w, e = a[1:-1, 1:-1], a[:-2, 1:-1], a[2:, 1:-1], a[1:-1, :-2], a[1:-1, 2:]
    out[1:-1, 1:-1] = 0.5 * c + 0.125 * (n + s + w + e)
    den[1:-1, 1:-1] = 0.5 * np.abs(c) + 0.125 * (np.abs(n) + np.abs(s) + np.abs(w) + np.abs(e))
    return out, den


def bf16_to_f64(bits: np.ndarray) -> np.ndarray:
    return (bits.astype(np.uint32) << 16).view(np.float32).astype(np.float64)


def gemm_bf16(a_bits: np.ndarray, b_bits: np.ndarray) -> np.ndarray:
    """C = A B^T from bf16 bit patterns, accumulated in fp64."""
    return bf16_to_f64(a_bits) @ bf16_to_f64(b_bits).T


def antt(shared, alone) -> float:
    """Average normalised turnaround time: mean(T_shared / T_alone)."""
    return float(np.mean(np.asarray(shared, np.float64) / np.asarray(alone, np.float64)))


def stp(shared, alone) -> float:
    """System throughput: sum(T_alone / T_shared)."""
    return float(np.sum(np.asarray(alone, np.float64) / np.asarray(shared, np.float64)))
