"""Diagnostic: chunked-scan resolution on long oracle-encoded windows (regular / irregular framing).
For each window size: scan stats, scan time, and on a fallback the first chunk whose entry matched no
candidate (its candidates and the previous chunk's chosen exit)."""
import ctypes as C
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle as O  # noqa: E402
from paper_conf_sc_eilingkkflm23_b200 import build, crk, gen  # noqa: E402

MiB = 1 << 20
build.build()
cfg = O.Config(prog=gen.PROG, vers=gen.VERS)


def stream(total, irregular, seed=1):
    g = gen.rng(seed)
    parts, n, i = [], 0, 0
    while n < total:
        d = gen.random_bytes(seed * 7 + i, gen.log_uniform_int(g, 1, 2 * MiB))
        L = O.call_header(0x200000 + i, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0) + \
            O.put_opaque_var(d.tobytes()) + O.put_u64(len(d))
        w = O.frame_lens(L, gen.split_points(seed * 131 + i, len(L))) if irregular else O.frame(L, 65536)
        parts.append(w)
        n += len(w)
        i += 1
    return b"".join(parts)


SumT = np.dtype([("start", "<u8"), ("exit", "<u8"), ("r0_after", "<u8"), ("sum_after", "<u8"), ("sum_total", "<u8"),
                 ("n", "<u4"), ("nlast", "<u4"), ("idx_last", "<i4"), ("kind", "<u4"), ("pad", "<u8")])
StT = np.dtype([("p", "<u8"), ("r0", "<u8"), ("sum", "<u8"), ("nf", "<u4"), ("nr", "<u4"), ("f0", "<u4"),
                ("chosen", "<i4"), ("skip", "<u4"), ("pad", "<u4")])

ctx = crk.Context(0)
for irr in (False, True):
    w = np.frombuffer(stream(int(os.environ.get("TOTAL_MIB", "256")) * MiB, irr), np.uint8)
    ring = crk.Ring.device(1 << 29)
    ring.tensor()[:len(w)].copy_(torch.from_numpy(w))
    for mib in (8, 32, 64, 128, 256):
        tail = min(len(w), mib * MiB)
        idx = ctx.index(1, 1 << 16, 1 << 12)
        idx.frame_scan([(ring, 0, tail)])
        torch.cuda.synchronize()
        st = idx.scan_stats()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        crk.profile_enable(True)
        e0.record()
        for _ in range(5):
            idx.frame_scan([(ring, 0, tail)])
        e1.record()
        torch.cuda.synchronize()
        prof = crk.profile_read()
        crk.profile_enable(False)
        print("  stage ms per launch:", {k: round(v[0] / max(1, v[1]), 4) for k, v in prof.items()})
        res = idx.ring_results(1)[0]
        print(f"irregular={irr} window={tail} stats={st} scan_ms={e0.elapsed_time(e1) / 5:.3f} "
              f"status={res['status']} frags={res['n_frags']}", flush=True)
        if st["fallback"]:
            ptrs = (C.c_void_p * 5)()
            cap = C.c_uint32()
            crk.lib().crk_debug_index_ms(idx.h, ptrs, C.byref(cap))
            K = 0
            # recompute the chunk plan's K from the sums (kind != 0 for chunk 0 cand 0)
            sums = crk.copy_to_host(ptrs[0], 64 * 4 * cap.value).view(SumT).reshape(cap.value, 4)
            state = crk.copy_to_host(ptrs[1], 48 * cap.value).view(StT)
            K = int(np.max(np.nonzero(sums["kind"][:, 0])[0])) + 1
            print("  K", K, "chosen", state["chosen"][:K].tolist()[:64])
            x = int(sums[0, 0]["exit"])
            for i in range(1, K):
                starts = [int(s) for s in sums[i]["start"]]
                if x not in starts:
                    print(f"  chunk {i}: entry {x} not in candidates {starts} kinds {sums[i]['kind'].tolist()} "
                          f"n {sums[i]['n'].tolist()}; prev chunk sums {sums[i - 1].tolist()}")
                    hv = w[x:x + 8]
                    print("  header at entry:", hv.tobytes().hex())
                    break
                j = starts.index(x)
                if sums[i, j]["kind"] != 1:
                    print(f"  chunk {i}: chain kind {sums[i, j]['kind']} n {sums[i, j]['n']}")
                    break
                x = int(sums[i, j]["exit"])
        del idx
