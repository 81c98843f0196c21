"""Pins for oracle/workloads.py against things other than itself: brute force on tiny inputs,
closed forms, special cases that reduce to a library routine."""
import numpy as np
import pytest
import scipy.sparse as sp

from oracle import workloads as W
from synth import gen


def _i32(v: int) -> int:
    v &= 0xFFFFFFFF
    return v - (1 << 32) if v >= (1 << 31) else v


def test_saxpy_i32_bruteforce_python_ints():
    x, y = gen.saxpy_i32_inputs(257, seed=5)
    for a in (0, 1, -1, 1664525, 22695477, -(2**31), 2**31 - 1):
        got = W.saxpy_i32(a, x, y)
        exp = [_i32(a * int(xi) + int(yi)) for xi, yi in zip(x, y)]
        assert got.dtype == np.int32
        assert got.tolist() == exp


def test_saxpy_i32_special_cases():
    x, y = gen.saxpy_i32_inputs(1000, seed=6)
    assert np.array_equal(W.saxpy_i32(0, x, y), y)
    assert np.array_equal(W.saxpy_i32(1, x, np.zeros_like(y)), x)
    # 2^16 * 2^16 = 2^32 wraps to 0
    assert W.saxpy_i32(65536, np.array([65536], np.int32), np.array([7], np.int32))[0] == 7
    # in-place update is non-idempotent: applying twice differs from once (exactly-once witness)
    once = W.saxpy_i32(3, x, y)
    twice = W.saxpy_i32(3, x, once)
    assert not np.array_equal(once, twice)


def test_saxpy_f32_special_cases():
    x, y = gen.saxpy_f32_inputs(1000, seed=7)
    assert np.array_equal(W.saxpy_f32(0.0, x, y), y.astype(np.float64))
    assert np.array_equal(W.saxpy_f32(1.0, x, np.zeros_like(y)), x.astype(np.float64))
    # a = 2, y = x -> 3x exactly (all fp32 values times 3 are exact in fp64)
    assert np.array_equal(W.saxpy_f32(2.0, x, x), 3.0 * x.astype(np.float64))


def test_spmv_matches_scipy_and_bruteforce():
    rowptr, col, val, x = gen.csr_inputs(300, seed=8)
    y, absum = W.spmv_csr(rowptr, col, val, x)
    A = sp.csr_matrix((val.astype(np.float64), col, rowptr), shape=(300, 300))
    assert np.allclose(y, A @ x.astype(np.float64), rtol=0, atol=1e-12)
    # dense brute force on a tiny matrix
    rowptr, col, val, x = gen.csr_inputs(9, seed=9, max_row_len=6)
    y, _ = W.spmv_csr(rowptr, col, val, x)
    for i in range(9):
        s = 0.0
        for p in range(rowptr[i], rowptr[i + 1]):
            s += float(val[p]) * float(x[col[p]])
        assert abs(y[i] - s) <= 1e-15 * max(1.0, abs(s))
    assert np.all(absum >= np.abs(W.spmv_csr(*gen.csr_inputs(300, seed=8))[0]) - 1e-12)


def test_spmv_identity_empty_rows_and_duplicates():
    n = 50
    rowptr = np.arange(n + 1, dtype=np.int32)
    col = np.arange(n, dtype=np.int32)
    val = np.ones(n, np.float32)
    x = gen.saxpy_f32_inputs(n, seed=10)[0]
    y, _ = W.spmv_csr(rowptr, col, val, x)
    assert np.array_equal(y, x.astype(np.float64))
    # empty rows -> 0; duplicate entries summed
    rowptr = np.array([0, 0, 3, 3], np.int32)
    col = np.array([1, 1, 2], np.int32)
    val = np.array([1.0, 2.0, 4.0], np.float32)
    x = np.array([5.0, 7.0, 0.5], np.float32)
    y, _ = W.spmv_csr(rowptr, col, val, x)
    assert y.tolist() == [0.0, 1 * 7 + 2 * 7 + 4 * 0.5, 0.0]


def test_csr_generator_structure():
    rowptr, col, val, x = gen.csr_inputs(1000, seed=2)
    lens = np.diff(rowptr)
    assert lens.min() >= 0 and lens.max() <= 20
    for i in range(0, 1000, 37):
        seg = col[rowptr[i]:rowptr[i + 1]]
        assert np.all(np.diff(seg) >= 0)


def test_stencil_f32_closed_forms_and_bruteforce():
    c = np.full((17, 23), 0.3125, np.float32)       # exact binary fraction
    out, _ = W.stencil5_f32(c)
    assert np.array_equal(out, c.astype(np.float64))
    i, j = np.meshgrid(np.arange(33), np.arange(40), indexing="ij")
    ramp = (i + j).astype(np.float32)
    out, _ = W.stencil5_f32(ramp)
    assert np.array_equal(out, ramp.astype(np.float64))   # harmonic: exact in the interior
    a = gen.stencil_f32_input(7, seed=3)
    out, absum = W.stencil5_f32(a)
    for r in range(7):
        for q in range(7):
            if r in (0, 6) or q in (0, 6):
                exp = float(a[r, q])
            else:
                exp = (0.5 * float(a[r, q]) + 0.125 * float(a[r - 1, q]) + 0.125 * float(a[r + 1, q])
                       + 0.125 * float(a[r, q - 1]) + 0.125 * float(a[r, q + 1]))
            assert abs(out[r, q] - exp) <= 1e-15
            assert absum[r, q] >= abs(out[r, q]) - 1e-15


def test_stencil_i32_closed_forms_and_bruteforce():
    c = np.full((9, 11), 123456789, np.int32)
    out = W.stencil5_i32(c)
    assert np.all(out[1:-1, 1:-1] == 0)
    assert np.array_equal(out[0], c[0]) and np.array_equal(out[:, -1], c[:, -1])
    a = gen.stencil_i32_input(6, seed=4)
    out = W.stencil5_i32(a)
    for r in range(1, 5):
        for q in range(1, 5):
            v = 4 * int(a[r, q]) - int(a[r - 1, q]) - int(a[r + 1, q]) - int(a[r, q - 1]) - int(a[r, q + 1])
            assert int(out[r, q]) == _i32(v)


def test_gemm_identity_ones_and_triple_loop():
    a_bits, b_bits = gen.gemm_bf16_inputs(8, 16, 16, seed=12)
    ident = gen.round_to_bf16_bits(np.eye(16, dtype=np.float32))
    c = W.gemm_bf16(a_bits, ident)
    assert np.array_equal(c, W.bf16_bits_to_f64(a_bits))
    ones = gen.round_to_bf16_bits(np.ones((4, 40), np.float32))
    assert np.all(W.gemm_bf16(ones, ones) == 40.0)
    a_bits, b_bits = gen.gemm_bf16_inputs(3, 5, 7, seed=13)
    c = W.gemm_bf16(a_bits, b_bits)
    A = W.bf16_bits_to_f64(a_bits)
    B = W.bf16_bits_to_f64(b_bits)
    for m in range(3):
        for n in range(5):
            s = 0.0
            for k in range(7):
                s += A[m, k] * B[n, k]
            assert c[m, n] == pytest.approx(s, abs=1e-14)
            assert W.gemm_entry(a_bits, b_bits, m, n) == pytest.approx(s, abs=1e-14)


def test_bf16_rounding_generator():
    v = np.array([1.0, 1.00390625, 1.005859375, -2.5, 3.0e38], np.float32)
    b = gen.round_to_bf16_bits(v)
    back = gen.bf16_bits_to_f32(b)
    assert back[0] == 1.0
    assert back[1] == 1.0              # tie -> even
    assert back[2] == 1.0078125        # above tie -> up
    assert back[3] == -2.5
