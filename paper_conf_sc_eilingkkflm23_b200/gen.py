"""Seeded synthetic workload generators.

This module holds NO XDR / record-marking arithmetic: it only draws the random quantities a workload
is made of (payload bytes, sizes, xids, item kinds and counts, fragment split points, destination
offsets) from numpy PCG64 streams.  Both the oracle (tests) and the CUDA path (bench, tests) consume
these descriptions and each encodes them with its own code.

Shapes follow the paper's workloads: matrixMul's transfers (§4.1; 1.95 MiB total),
bandwidthTest's HtoD/DtoH sweep up to 512 MiB (§4.2), plus the stress and
multi-endpoint configs BASELINE.json names.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

KiB, MiB, GiB = 1 << 10, 1 << 20, 1 << 30

# Item kind names used by workload descriptions.  The numeric codes are the interface codes of
# DESIGN.md §4 (include/crk.h CRK_K_*), spelled out here so descriptions can be handed to either side.
U32, U64, OPAQUE_VAR, OPAQUE_FIX = 1, 2, 3, 4
I32_VAR, U32_VAR, F32_VAR, I64_VAR, U64_VAR, F64_VAR = 5, 6, 7, 8, 9, 10
I32_FIX, U32_FIX, F32_FIX, I64_FIX, U64_FIX, F64_FIX = 11, 12, 13, 14, 15, 16
NP_DTYPE = {I32_VAR: np.int32, U32_VAR: np.uint32, F32_VAR: np.float32, I64_VAR: np.int64,
            U64_VAR: np.uint64, F64_VAR: np.float64, I32_FIX: np.int32, U32_FIX: np.uint32,
            F32_FIX: np.float32, I64_FIX: np.int64, U64_FIX: np.uint64, F64_FIX: np.float64}

# Test/bench RPC program constants (reading R15: arbitrary, NOT Cricket's numbers).
PROG, VERS, PROC_H2D, PROC_D2H = 0x20000099, 1, 1, 2
PROC_C1 = 7
F_DEFAULT = 65536


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def random_bytes(seed: int, n: int) -> np.ndarray:
    return rng(seed).integers(0, 256, size=n, dtype=np.uint8)


def log_uniform_int(g: np.random.Generator, lo: int, hi: int) -> int:
    return int(round(math.exp(g.uniform(math.log(lo), math.log(hi)))))


def split_points(seed: int, total: int, lo: int = 1, hi: int = 65536) -> list[int]:
    """Fragment lengths uniform in [lo, hi] summing to total (C4-ii irregular framing)."""
    g = rng(seed)
    out, left = [], total
    while left > 0:
        x = min(left, int(g.integers(lo, hi + 1)))
        out.append(x)
        left -= x
    return out or [0]


def special_bits(dtype) -> np.ndarray:
    """Bit patterns every typed-array test must carry through unchanged."""
    if dtype in (np.float32,):
        u = np.array([0x7FC00000, 0x7FA00001, 0xFFC12345, 0x7F800001, 0x7F800000, 0xFF800000, 0x00000000,
                      0x80000000, 0x00000001, 0x807FFFFF, 0x3F800000], np.uint32)
        return u.view(np.float32)
    if dtype in (np.float64,):
        u = np.array([0x7FF8000000000000, 0x7FF4000000000001, 0xFFF8123456789ABC, 0x7FF0000000000001,
                      0x7FF0000000000000, 0xFFF0000000000000, 0, 0x8000000000000000, 1, 0x800FFFFFFFFFFFFF,
                      0x3FF0000000000000], np.uint64)
        return u.view(np.float64)
    info = np.iinfo(dtype)
    return np.array([info.min, info.max, 0, 1, -1 if info.min < 0 else info.max - 1], dtype=dtype)


def random_elems(g: np.random.Generator, dtype, count: int) -> np.ndarray:
    """Uniform random bit patterns of `dtype` with the special values spliced in."""
    es = np.dtype(dtype).itemsize
    raw = g.integers(0, 256, size=count * es, dtype=np.uint8).view(dtype).copy()
    sp = special_bits(dtype)
    k = min(len(sp), count)
    if k:
        pos = g.choice(count, size=k, replace=False)
        raw[pos] = sp[:k]
    return raw


@dataclass
class Call:
    """One CALL record: proc, xid and its argument items as (kind, value) in schema order.
    Opaque values are uint8 arrays, array values numpy arrays of the kind's dtype, scalars ints."""
    xid: int
    proc: int
    items: list
    frag_lens: list | None = None  # explicit framing; None = greedy with the config's F


# ------------------------------------------------------------------ C1: one single-fragment record

C1_SCHEMA = [U64, OPAQUE_VAR, U64, I32_VAR]


def c1_call(xid: int = 0xC1C1C1C1, ptr: int = 0x7F0000001000) -> Call:
    data = random_bytes(0xC1, 4096)
    ints = rng(0xC1 + 1).integers(-(1 << 31), 1 << 31, size=1024, dtype=np.int64).astype(np.int32)
    return Call(xid, PROC_C1, [(U64, ptr), (OPAQUE_VAR, data), (U64, 4096), (I32_VAR, ints)])


# ------------------------------------------------------------------ C2: matrixMul transfers

def c2_matrices():
    """CUDA Samples matrixMul dims (A 320x320, B 640x320 with width 640 -> C 640x320 floats):
    A = 1.0f, B = 0.01f, C = 320 * 0.01f = 3.2f.  Sum = 2,048,000 B = 1.953 MiB."""
    A = np.full(320 * 320, 1.0, np.float32)
    B = np.full(640 * 320, 0.01, np.float32)
    C = np.full(640 * 320, np.float32(320) * np.float32(0.01), np.float32)
    return A, B, C


# ------------------------------------------------------------------ C3: bandwidth sweep

C3_LOG2 = list(range(12, 31))  # 4 KiB .. 1 GiB; 2^29 is the paper's 512 MiB point


def c3_payload(log2n: int) -> np.ndarray:
    return random_bytes(0xC3 + log2n, 1 << log2n)


# ------------------------------------------------------------------ C4: typed-array stress

C4_SCHEMAS = {
    10: [OPAQUE_VAR, I32_VAR],
    11: [U64_VAR, F32_VAR, F64_VAR],
    12: [OPAQUE_VAR, OPAQUE_VAR, F64_VAR],
    13: [I32_VAR],
    14: [F32_VAR, OPAQUE_VAR, U64_VAR, I32_VAR],
    15: [F64_VAR, U32, OPAQUE_VAR],
    16: [U64, I64_VAR, U32_VAR, OPAQUE_VAR, F32_VAR],
    17: [OPAQUE_FIX | (13 << 8), I32_FIX | (7 << 8), F64_VAR],
}


def c4_calls(total_bytes: int, seed: int = 0xC4, max_count: int = 1 << 20,
             xid0: int = 0x40000000) -> list[Call]:
    """Records of random item sequences until `total_bytes` of item payload exist.  Opaque lengths
    are odd (pad 1 or 3); counts log-uniform in [1, max_count]."""
    g = rng(seed)
    procs = sorted(C4_SCHEMAS)
    calls, total, xid = [], 0, xid0
    while total < total_bytes:
        proc = int(g.choice(procs))
        items = []
        for code in C4_SCHEMAS[proc]:
            kind, fixed = code & 0xFF, code >> 8
            if kind == U32:
                items.append((kind, int(g.integers(0, 1 << 32))))
            elif kind == U64:
                items.append((kind, int(g.integers(0, 1 << 63)) * 2 + int(g.integers(0, 2))))
            elif kind in (OPAQUE_VAR, OPAQUE_FIX):
                n = fixed if kind == OPAQUE_FIX else log_uniform_int(g, 1, max_count) | 1
                items.append((kind, g.integers(0, 256, size=n, dtype=np.uint8)))
                total += n
            else:
                n = fixed if fixed else log_uniform_int(g, 1, max_count)
                arr = random_elems(g, NP_DTYPE[kind], n)
                items.append((kind, arr))
                total += arr.nbytes
        calls.append(Call(xid, proc, items))
        xid += 1
    return calls


def frag_seed(call: Call) -> int:
    """Seed of the C4-ii irregular split of `call`: the encoder side asks split_points(frag_seed(c), L)
    for its own logical length L."""
    return (0xC4 + 1) ^ (call.xid * 0x9E3779B1 & 0xFFFFFFFF)


# ------------------------------------------------------------------ C5: per-GPU endpoint streams

@dataclass
class MemcpyRec:
    kind: int        # PROC_H2D or PROC_D2H
    xid: int
    size: int        # payload bytes
    region_off: int  # offset of dst (HtoD) / src (DtoH) inside the endpoint's device region
    seed: int        # payload seed (HtoD data, or the DtoH source contents)


@dataclass
class Stream:
    gpu: int
    stream: int
    records: list = field(default_factory=list)


def c5_endpoint(gpu: int, n_streams: int = 16, payload_per_stream: int = 64 * MiB, h2d_budget: int = 60 * MiB,
                lo: int = 4 * KiB, hi: int = 16 * MiB, h2d_frac: float = 0.5, align: int = 256,
                misalign: bool = False) -> tuple[list[Stream], int]:
    """The streams of one endpoint (one GPU) and the size of the device region their pointers name.
    Sizes are log-uniform in [lo, hi]; each stream carries `payload_per_stream` payload bytes, at most
    `h2d_budget` of them HtoD (so its receive ring stays within the caller's capacity).  HtoD
    destinations and DtoH sources get disjoint region ranges (a serve batch is concurrent)."""
    streams, off = [], 0
    for s in range(n_streams):
        seed = (0xC5 << 8) | (gpu << 4) | s
        g = rng(seed)
        st = Stream(gpu, s)
        payload, h2d, seq = 0, 0, 0
        while payload < payload_per_stream:
            size = max(1, min(log_uniform_int(g, lo, hi), payload_per_stream - payload))
            kind = PROC_H2D if g.random() < h2d_frac else PROC_D2H
            if kind == PROC_H2D and h2d + size > h2d_budget:
                kind = PROC_D2H
            shift = int(g.integers(0, 16)) if misalign else 0
            st.records.append(MemcpyRec(kind, (gpu << 28) | (s << 20) | seq, size, off + shift,
                                        int(g.integers(0, 1 << 62))))
            off = (off + shift + size + align - 1) // align * align
            payload += size
            h2d += size if kind == PROC_H2D else 0
            seq += 1
        streams.append(st)
    return streams, off


# ------------------------------------------------------------------ NEXT-2: more of the paper's workloads

# cuSolverDn_LinearSolver: "LU with 900x900 matrix, 1000 Iterations" (Fig. 5b), 6.07 GiB of
# memory transfers in all.  Per iteration the sample copies the matrix A (n x n doubles) and
# the right-hand side b (n doubles) to the device and the solution x (n doubles) back; 1000 iterations move
# 6,494,400,000 B = 6.05 GiB (the paper's 6.07 GiB also counts the sample's setup copies).
CUSOLVER_N, CUSOLVER_ITERS = 900, 1000
# histogram: 64 MiB of memory transfers: the CUDA sample's 64 MiB byte array to the device and
# its 256-bin uint32 histogram back.
HISTOGRAM_BYTES, HISTOGRAM_BINS = 64 * MiB, 256


def _profile_streams(recs_per_stream: list[list[tuple[int, int]]], gpu: int, seed: int,
                     align: int = 256) -> tuple[list[Stream], int]:
    """Streams of (kind, size) memcpy calls laid out in one region (disjoint, `align`-aligned ranges)."""
    g = rng(seed)
    streams, off = [], 0
    for s, recs in enumerate(recs_per_stream):
        st = Stream(gpu, s)
        for seq, (kind, size) in enumerate(recs):
            st.records.append(MemcpyRec(kind, (gpu << 28) | (s << 20) | seq, size, off, int(g.integers(0, 1 << 62))))
            off = (off + size + align - 1) // align * align
        streams.append(st)
    return streams, off


def cusolver_endpoint(gpu: int = 0, iterations: int = CUSOLVER_ITERS, n: int = CUSOLVER_N, n_streams: int = 1,
                      seed: int = 0xC50D) -> tuple[list[Stream], int]:
    """cuSolverDn_LinearSolver's memcpy calls: per iteration A (n*n*8 B) and b (n*8 B) HtoD, x (n*8 B) DtoH,
    iterations dealt round-robin over n_streams client streams (one stream = one connection)."""
    per = [[] for _ in range(n_streams)]
    for it in range(iterations):
        per[it % n_streams] += [(PROC_H2D, n * n * 8), (PROC_H2D, n * 8), (PROC_D2H, n * 8)]
    return _profile_streams(per, gpu, seed)


def histogram_endpoint(gpu: int = 0, nbytes: int = HISTOGRAM_BYTES, bins: int = HISTOGRAM_BINS,
                       seed: int = 0x4157) -> tuple[list[Stream], int]:
    """histogram's memcpy calls: the byte array HtoD, the bins (uint32) DtoH, on one client stream."""
    return _profile_streams([[(PROC_H2D, nbytes), (PROC_D2H, bins * 4)]], gpu, seed)
