"""Seeded input generators (NumPy PCG64). See DESIGN.md "Input recipe" for the table.

Every generator is a pure function of its arguments (seed included). Nothing here computes a
workload result, a coverage set or a scheduling decision.
"""
from __future__ import annotations

import numpy as np

__all__ = [
    "rng",
    "saxpy_i32_inputs",
    "saxpy_f32_inputs",
    "csr_inputs",
    "stencil_f32_input",
    "stencil_i32_input",
    "round_to_bf16_bits",
    "bf16_bits_to_f32",
    "gemm_bf16_inputs",
    "preempt_schedule",
    "queue_trace",
    "SAXPY_BLOCK",
    "SPMV_ROWS_PER_BLOCK",
    "STENCIL_TILE",
    "GEMM_TILE_M",
    "GEMM_TILE_N",
]

# Original-kernel block geometry (the "task" of P:128/P:164). Fixed by DESIGN.md.
SAXPY_BLOCK = 256          # elements per original CTA (CUDA SDK vectorAdd: one element per thread)
SPMV_ROWS_PER_BLOCK = 128  # rows per original CTA (CSR-stream block of 256 threads)
STENCIL_TILE = 64          # 64x64 output cells per original CTA
GEMM_TILE_M = 128          # output tile rows per original CTA
GEMM_TILE_N = 256          # output tile cols per original CTA


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def saxpy_i32_inputs(n: int, seed: int):
    """x, y uniform over the full int32 range (config 1: seed 1 for LP, seed 11 for HP)."""
    g = rng(seed)
    x = g.integers(-(2**31), 2**31, size=n, dtype=np.int64).astype(np.int32)
    y = g.integers(-(2**31), 2**31, size=n, dtype=np.int64).astype(np.int32)
    return x, y


def saxpy_f32_inputs(n: int, seed: int):
    """x, y uniform on [-1, 1) in fp32."""
    g = rng(seed)
    x = g.uniform(-1.0, 1.0, size=n).astype(np.float32)
    y = g.uniform(-1.0, 1.0, size=n).astype(np.float32)
    return x, y


def csr_inputs(rows: int, seed: int, max_row_len: int = 20, cols: int | None = None,
               empty_runs=()):
    """CSR matrix with row length uniform in {0..max_row_len}, columns uniform with replacement
    and sorted within each row (duplicates allowed), val and x uniform on [-1, 1) fp32.
    SURVEY §8(c) A28 / §8(d) C2 (1M rows, ~10.5M nnz at seed 2). `empty_runs` = [(r0, r1), ...]
    forces rows r0..r1-1 empty (edge-case inputs: whole empty row groups)."""
    g = rng(seed)
    ncols = rows if cols is None else cols
    lens = g.integers(0, max_row_len + 1, size=rows, dtype=np.int64)
    for r0, r1 in empty_runs:
        lens[r0:r1] = 0
    rowptr = np.zeros(rows + 1, dtype=np.int64)
    np.cumsum(lens, out=rowptr[1:])
    nnz = int(rowptr[-1])
    c = g.integers(0, ncols, size=nnz, dtype=np.int64)
    row_id = np.repeat(np.arange(rows, dtype=np.int64), lens)
    key = row_id * ncols + c
    key.sort()
    col = (key % ncols).astype(np.int32)
    val = g.uniform(-1.0, 1.0, size=nnz).astype(np.float32)
    x = g.uniform(-1.0, 1.0, size=ncols).astype(np.float32)
    return rowptr.astype(np.int32), col, val, x


def stencil_f32_input(n: int, seed: int):
    """n x n field, uniform [0, 1) fp32, row-major."""
    return rng(seed).uniform(0.0, 1.0, size=(n, n)).astype(np.float32)


def stencil_i32_input(n: int, seed: int):
    """n x n field, uniform over the full int32 range, row-major."""
    return rng(seed).integers(-(2**31), 2**31, size=(n, n), dtype=np.int64).astype(np.int32)


def round_to_bf16_bits(a: np.ndarray) -> np.ndarray:
    """fp32 -> bf16 bit patterns (uint16), round-to-nearest-even. Input finite."""
    u = np.ascontiguousarray(a, dtype=np.float32).view(np.uint32).astype(np.uint64)
    bias = ((u >> 16) & 1) + 0x7FFF
    return ((u + bias) >> 16).astype(np.uint16)


def bf16_bits_to_f32(b: np.ndarray) -> np.ndarray:
    return (b.astype(np.uint32) << 16).view(np.float32)


def gemm_bf16_inputs(m: int, n: int, k: int, seed: int):
    """A [m,k] row-major and B [n,k] row-major (K-major, "TN"), bf16 bit patterns of
    uniform [-1, 1) values. Returns (A_bits, B_bits)."""
    g = rng(seed)
    a = g.uniform(-1.0, 1.0, size=(m, k)).astype(np.float32)
    b = g.uniform(-1.0, 1.0, size=(n, k)).astype(np.float32)
    return round_to_bf16_bits(a), round_to_bf16_bits(b)


def preempt_schedule(seed: int, n_blocks: int, num_sms: int):
    """One random manual-mode preempt/resume schedule for config 1:
    1-4 cycles; each cycle a trigger block t* and a yield width n (temporal = num_sms, or
    spatial uniform in [1, num_sms-1]); chunk C and poll period K.
    Returns dict(C, K, cycles=[(t_star, n_sms), ...]) with t_star strictly increasing."""
    g = rng(seed)
    C = int(g.choice([1, 2, 4, 8, 16]))
    K = int(g.choice([1, 2, 4, 8]))
    ncyc = int(g.integers(1, 5))
    ts = np.sort(g.choice(np.arange(1, max(2, n_blocks)), size=min(ncyc, max(1, n_blocks - 1)), replace=False))
    cycles = []
    for t in ts:
        if g.random() < 0.5:
            nsm = num_sms
        else:
            nsm = int(g.integers(1, num_sms))
        cycles.append((int(t), nsm))
    return {"C": C, "K": K, "cycles": cycles}


# Size classes of config 4, mirroring Table 1's trivial/small/large ratios.
QUEUE_SIZES = {
    "saxpy_f32": [2**20, 2**24, 2**28],            # elements
    "spmv": [2**16, 2**20, 2**23],                 # rows
    "stencil_f32": [1024, 4096, 16384],            # n (n x n)
    "gemm_bf16": [2048, 4096, 8192],               # M = N = K
}


def queue_trace(seed: int, n_kernels: int, mean_gap_ns: int, burst: bool = False,
                types=("saxpy_f32", "spmv", "stencil_f32", "gemm_bf16")):
    """Mixed same-priority queue (config 4/5): type uniform over `types`, size class uniform
    over {0: trivial, 1: small, 2: large}, Poisson arrivals with the given mean gap (or all at
    t=0 when burst). Returns a list of dicts sorted by arrival time."""
    g = rng(seed)
    out = []
    t = 0
    for i in range(n_kernels):
        ty = types[int(g.integers(0, len(types)))]
        cls = int(g.integers(0, 3))
        if not burst and i > 0:
            t += int(g.exponential(mean_gap_ns))
        out.append({"id": i, "type": ty, "size_class": cls, "size": QUEUE_SIZES[ty][cls],
                    "arrival_ns": 0 if burst else t, "priority": 0})
    return out
