"""Diagnostic: per-phase times of the chunked scan's K1a CTAs (build variant with -DCRK_MSCAN_TRACE) on a
C3-shaped 1 GiB record and a C4-ii irregular 256 MiB stream.  Prints, per phase, the median and max over CTAs
of its duration and the spread of CTA start times."""
import ctypes as C
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle as O  # noqa: E402
from paper_conf_sc_eilingkkflm23_b200 import build, crk, gen  # noqa: E402

MiB = 1 << 20
crk.LIBPATH = build.build_variant("mtrace", ["CRK_MSCAN_TRACE"])
L = crk.lib()
L.crk_debug_mscan_trace.argtypes = [C.c_void_p]
ctx = crk.Context(0)
names = ["zone", "hop1", "score", "select", "walk", "resolve"]
from paper_conf_sc_eilingkkflm23_b200 import workload  # noqa: E402
for label, mib in (("8MiB", 8), ("1GiB", 1024), ("C5", 0)):
    if label == "C5":  # the bench endpoint: 16 rings, mixed HtoD / DtoH memcpy CALLs
        ep = workload.c5_endpoint(ctx, 0, torch.device("cuda:0"))
        rings = ep.rings
        idx = ctx.index(16, 1 << 20, 1 << 14)
    else:
        n = mib * MiB
        payload = gen.c3_payload(30)[:n]
        Lr = O.call_header(0xC3, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0) + O.put_u32(n)
        w = np.frombuffer(O.frame(Lr + payload.tobytes() + O.put_u64(n), 65536), np.uint8)
        ring = crk.Ring.device(1 << 31)
        ring.tensor()[:len(w)].copy_(torch.from_numpy(w.copy()))
        idx = ctx.index(1, 1 << 15, 16)
        rings = [(ring, 0, len(w))]
    for _ in range(3):
        idx.frame_scan(rings)
    torch.cuda.synchronize()
    buf = np.zeros((4096, 12), np.uint64)
    L.crk_debug_mscan_trace(buf.ctypes.data)
    k = int(idx.scan_stats()["chunked"])
    used = buf[:, 0] > 0
    t = buf[used].astype(np.int64)
    t = t[t[:, 6] > 0]
    t0 = t[:, 0].min()
    print(label, "ctas", len(t), "stats", idx.scan_stats(), "span us", (t[:, 6].max() - t0) / 1e3)
    print("  start spread us", np.percentile((t[:, 0] - t0) / 1e3, [50, 90, 100]).round(1).tolist())
    for p in range(1, 7):
        d = (t[:, p] - t[:, p - 1]) / 1e3
        d = d[t[:, p - 1] > 0]
        print(f"  {names[p - 1]:8s} median {np.median(d):7.2f} max {d.max():7.2f} us")
    last = t[np.argmax(t[:, 6])]  # the resolving CTA: its sub-phases
    print("  resolver: stage %.2f  maps %.2f  map-scan %.2f  chosen-sums %.2f  scans %.2f  states %.2f us" % tuple(
        (last[b] - last[a]) / 1e3 for a, b in ((5, 7), (7, 11), (11, 8), (8, 9), (9, 10), (10, 6))))
    # candidate summary per chunk (sums of the last launch)
    ptrs = (C.c_void_p * 5)()
    cap = C.c_uint32()
    L.crk_debug_index_ms(idx.h, ptrs, C.byref(cap))
    SumT = np.dtype([("start", "<u8"), ("exit", "<u8"), ("r0_after", "<u8"), ("sum_after", "<u8"),
                     ("sum_total", "<u8"), ("n", "<u4"), ("nlast", "<u4"), ("idx_last", "<i4"), ("kind", "<u4"),
                     ("pad", "<u8")])
    sums = crk.copy_to_host(ptrs[0], 64 * 4 * cap.value).view(SumT).reshape(cap.value, 4)[:len(t)]
    nc = (sums["kind"] != 0).sum(1)
    print("  candidates per chunk:", np.bincount(nc).tolist(), "kinds:", np.bincount(sums["kind"].ravel()).tolist())
    del rings, idx
    torch.cuda.empty_cache()
