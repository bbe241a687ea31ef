"""Mutation fuzzing of the chunked multi-CTA scan (k_mscan.cu) against the oracle's or_frame_scan: long windows
(2-6 MiB, so they are cut into chunks) of valid memcpy CALL streams -- greedy 64 KiB framing, irregular framing,
tiny records between big ones -- with seeded header rewrites (lengths, last bits, zero-length fragments),
byte flips, spliced garbage, dropped bytes and truncations placed anywhere, including at and around chunk
boundaries.  Every ring's status, consumed cursor, fragment table and record table must equal the oracle's;
the fallback to the one-CTA scan is allowed (and counted), a wrong answer is not."""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import gen
from tests.gpu_util import compare_scan, ctx_for, d2h_call, h2d_call, make_ring, ocfg, ring_np

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("needs a GPU", allow_module_level=True)

MiB = 1 << 20


def base_stream(g, cfg, total):
    parts, n, i = [], 0, 0
    while n < total:
        k = int(g.integers(0, 4))
        if k == 0:  # a big HtoD, greedy framing
            size = gen.log_uniform_int(g, 4096, 2 * MiB)
            w = O.encode_call(*h2d_call(i, gen.random_bytes(i + 1, size)), cfg)
        elif k == 1:  # irregular framing
            size = gen.log_uniform_int(g, 1, MiB)
            L = O.call_header(i, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0) + \
                O.put_opaque_var(gen.random_bytes(i + 2, size).tobytes()) + O.put_u64(size)
            w = O.frame_lens(L, gen.split_points(i * 7 + 3, len(L), 1, 65536))
        else:  # small DtoH CALLs
            w = b"".join(O.encode_call(*d2h_call(i * 16 + j, 0x7F0000000000, 4096), cfg)
                         for j in range(int(g.integers(1, 20))))
        parts.append(w)
        n += len(w)
        i += 1
    return bytearray(b"".join(parts))


def mutate(g, w, S):
    for _ in range(int(g.integers(1, 4))):
        near_boundary = g.random() < 0.5
        pos = (int(g.integers(1, max(2, len(w) // S))) * S + int(g.integers(-70000, 70000))) if near_boundary \
            else int(g.integers(0, len(w)))
        pos = min(max(pos, 0), len(w) - 1)
        kind = int(g.integers(0, 5))
        if kind == 0:
            w[pos] ^= int(g.integers(1, 256))
        elif kind == 1:  # a field rewrite: record-mark lengths / last bits, zero-length fragments
            w[pos:pos + 4] = int(g.choice([0, 0x80000000, 0x00010000, 0x80010000, 0x0000FFFF, 0x7FFFFFFF, 60,
                                           0x8000003C])).to_bytes(4, "big")
        elif kind == 2:
            w[pos:pos] = bytes(gen.random_bytes(pos, int(g.integers(1, 40))))
        elif kind == 3:
            del w[pos:pos + int(g.integers(1, 16))]
        else:
            del w[pos:]
    return bytes(w)


@pytest.mark.parametrize("seed", range(int(__import__("os").environ.get("CHUNK_FUZZ_SEEDS", "24"))))
def test_mutated_long_windows_match_oracle(seed):
    g = gen.rng(1000 + seed)
    cfg = ocfg()
    ctx = ctx_for(cfg, max_record_bytes=int(g.choice([1 << 32, 3 * MiB])))
    total = int(g.integers(2, 7)) * MiB
    w = mutate(g, base_stream(g, cfg, total), 256 * 1024)
    head = int(g.integers(0, 1 << 20))
    ring = make_ring(1 << 23)
    ring.write(head, w)
    idx = ctx.index(1, 1 << 16, 1 << 12)
    idx.frame_scan([(ring, head, head + len(w))])
    T = idx.tables()
    s = compare_scan(T, 0, ring_np(ring), head, head + len(w), 1 << 16, 1 << 12,
                     max_record_bytes=ctx.cfg.max_record_bytes)
    st = idx.scan_stats()  # windows a truncation left shorter than two chunks take the one-CTA scan
    assert st["chunked"] + st["fallback"] == (1 if len(w) >= 2 * 256 * 1024 else 0), (len(w), st)
