"""Plain definitions of the workload kernels (the "original kernel" bodies FLEP wraps).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py). FLEP's result is exactly the result of
running every original block once ("resume ... to finish the remaining tasks", P:164,
P:176), so the oracle for each workload is its plain mathematical definition, computed
without any notion of blocks, preemption or chunks. Floating point is computed in fp64
(SURVEY §8(c) O1b-O1f); integer work wraps modulo 2^32 in two's complement (A26).
"""
from __future__ import annotations

import numpy as np

_MASK32 = (1 << 32) - 1


def _wrap_i32(v: np.ndarray) -> np.ndarray:
    """Reduce int64 values modulo 2^32 into two's-complement int32."""
    return (v.astype(np.int64) & _MASK32).astype(np.uint32).view(np.int32)


def saxpy_i32(a: int, x: np.ndarray, y: np.ndarray) -> np.ndarray:
    """O1a — VA-shaped kernel (Table 1; BJ "SAXPY-int"): y'[i] = (a*x[i] + y[i]) mod 2^32.

    a*x fits in int64 (|a|,|x| < 2^31), and so does a*x + y, so the int64 sum is exact
    before the wrap."""
    a64 = np.int64(np.int32(a))
    return _wrap_i32(a64 * x.astype(np.int64) + y.astype(np.int64))


def saxpy_f32(a: float, x: np.ndarray, y: np.ndarray) -> np.ndarray:
    """O1b — y' = a*x + y in fp64 from fp32 inputs."""
    return np.float64(np.float32(a)) * x.astype(np.float64) + y.astype(np.float64)


def spmv_csr(rowptr: np.ndarray, col: np.ndarray, val: np.ndarray, x: np.ndarray):
    """O1c — SPMV: y[i] = sum_{p=rowptr[i]}^{rowptr[i+1]-1} val[p]*x[col[p]],
    fp64. Empty rows give 0; duplicate column entries are summed (each is a separate term).

    Returns (y, absum) where absum[i] = sum_p |val[p]*x[col[p]]| is the cancellation-safe
    tolerance denominator of SURVEY §8(c) "Parity criteria"."""
    rows = rowptr.shape[0] - 1
    lens = np.diff(rowptr.astype(np.int64))
    row_of = np.repeat(np.arange(rows, dtype=np.int64), lens)
    prod = val.astype(np.float64) * x.astype(np.float64)[col.astype(np.int64)]
    y = np.zeros(rows, dtype=np.float64)
    absum = np.zeros(rows, dtype=np.float64)
    np.add.at(y, row_of, prod)
    np.add.at(absum, row_of, np.abs(prod))
    return y, absum


# 5-point stencil weights: exact binary fractions.
W_C = 0.5
W_N = W_S = W_W = W_E = 0.125


def stencil5_f32(a: np.ndarray):
    """O1d — out-of-place 5-point sweep, fp64:
    interior out[i][j] = 0.5*in[i][j] + 0.125*(in[i-1][j] + in[i+1][j] + in[i][j-1] + in[i][j+1]);
    boundary rows and columns are copied through (out = in).

    Returns (out, absum) with absum = sum of |w*in| over the five terms (boundary: |in|)."""
    a = a.astype(np.float64)
    out = a.copy()
    absum = np.abs(a).copy()
    c = a[1:-1, 1:-1]
    n = a[:-2, 1:-1]
    s = a[2:, 1:-1]
    w = a[1:-1, :-2]
    e = a[1:-1, 2:]
    out[1:-1, 1:-1] = W_C * c + W_N * n + W_S * s + W_W * w + W_E * e
    absum[1:-1, 1:-1] = (W_C * np.abs(c) + W_N * np.abs(n) + W_S * np.abs(s)
                         + W_W * np.abs(w) + W_E * np.abs(e))
    return out, absum


def stencil5_i32(a: np.ndarray) -> np.ndarray:
    """O1e — integer 5-point sweep: interior out = (4*c - n - s - w - e) mod 2^32;
    boundary copied through. Exact in int64 before the wrap (|terms| < 2^34)."""
    a64 = a.astype(np.int64)
    out = a64.copy()
    out[1:-1, 1:-1] = (4 * a64[1:-1, 1:-1] - a64[:-2, 1:-1] - a64[2:, 1:-1]
                       - a64[1:-1, :-2] - a64[1:-1, 2:])
    return _wrap_i32(out)


def bf16_bits_to_f64(bits: np.ndarray) -> np.ndarray:
    """Decode bf16 bit patterns exactly (bf16 = upper half of an fp32)."""
    return (bits.astype(np.uint32) << 16).view(np.float32).astype(np.float64)


def gemm_bf16(a_bits: np.ndarray, b_bits: np.ndarray) -> np.ndarray:
    """O1f — MM: C[m][n] = sum_k A[m][k]*B[n][k] (C = A·Bᵀ, B stored N×K,
    K-major), from bf16-valued inputs, accumulated in fp64 (the products of two bf16 values
    are exact in fp64)."""
    a = bf16_bits_to_f64(a_bits)
    b = bf16_bits_to_f64(b_bits)
    return a @ b.T


def gemm_entry(a_bits: np.ndarray, b_bits: np.ndarray, m: int, n: int) -> float:
    """One output element of O1f, computed on its own (for sampled checks at full size)."""
    a = bf16_bits_to_f64(a_bits[m])
    b = bf16_bits_to_f64(b_bits[n])
    return float(np.dot(a, b))
