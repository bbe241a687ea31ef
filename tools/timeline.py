"""Per-stage timeline of small server steps from the diagnostic build's %globaltimer stamps
(-DCRK_TIMELINE -> lib/libcrk_timeline.so): for each stage, start and end (ns) relative to the step's first
kernel start, median over repetitions, plus the CUDA-event time of the whole step.

  python tools/timeline.py [--reps 200]
"""
import argparse
import ctypes as C
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_sc_eilingkkflm23_b200 import build  # noqa: E402

os.environ["CRK_LIB"] = build.build_variant("timeline", ["CRK_TIMELINE"])

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_sc_eilingkkflm23_b200 import crk, gen  # noqa: E402

STAGES = ["scan", "parse", "plan", "move", "fused", "m5", "m6", "m7"]


def run(case, ctx, fn, reps):
    L = crk.lib()
    L.crk_debug_timeline.restype = C.c_int
    L.crk_debug_timeline.argtypes = [C.c_void_p, C.c_void_p]
    tl = torch.zeros(16, dtype=torch.int64, device="cuda")
    L.crk_debug_timeline(ctx.h, tl.data_ptr())
    rows = []
    for _ in range(reps):
        tl.view(8, 2)[:, 0] = 0x7FFFFFFFFFFFFFFF
        tl.view(8, 2)[:, 1] = 0
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        t = tl.view(8, 2).cpu().numpy()
        rows.append((t, e0.elapsed_time(e1) * 1e3))
    L.crk_debug_timeline(ctx.h, None)
    out = {"case": case, "event_us_median": round(float(np.median([r[1] for r in rows])), 2)}
    t0s = [min(int(r[0][i, 0]) for i in range(5) if r[0][i, 1]) for r in rows]
    for i, name in enumerate(STAGES):
        if not any(r[0][i, 1] for r in rows):
            continue
        if i >= 5:  # end-only markers
            en = [int(r[0][i, 1]) - t0 for r, t0 in zip(rows, t0s)]
            out[name] = {"at_us": round(float(np.median(en)) / 1e3, 2)}
            continue
        st = [int(r[0][i, 0]) - t0 for r, t0 in zip(rows, t0s)]
        en = [int(r[0][i, 1]) - t0 for r, t0 in zip(rows, t0s)]
        out[name] = {"start_us": round(float(np.median(st)) / 1e3, 2), "end_us": round(float(np.median(en)) / 1e3, 2)}
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=200)
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    res = []
    # one 4 KiB HtoD CALL (C1-like)
    ctx = crk.Context(0)
    region = torch.zeros(1 << 20, dtype=torch.uint8, device=dev)
    base = region.data_ptr()
    data = torch.from_numpy(gen.random_bytes(0xC1, 4096)).to(dev)
    ring = crk.Ring.device(1 << 14)
    w = ctx.encode_call(7, gen.PROC_H2D, [(crk.K_U64, base + 4096), (crk.K_OPAQUE_VAR, data), (crk.K_U64, 4096)],
                        ring, 0)
    send = crk.Ring.device(1 << 12)
    idx = ctx.index(1, 64, 16)
    res.append(run("serve 1 x 4 KiB HtoD", ctx, lambda: idx.serve([(ring, 0, w)], [send], [0], base, region.numel()),
                   a.reps))
    # C2 matrixMul batch
    A, B, Cm = gen.c2_matrices()
    region2 = torch.zeros(4 << 20, dtype=torch.uint8, device=dev)
    b2 = region2.data_ptr()
    ta, tb = torch.from_numpy(A.view(np.uint8)).to(dev), torch.from_numpy(B.view(np.uint8)).to(dev)
    ring2 = crk.Ring.device(1 << 21)
    cur = ctx.encode_call(1, gen.PROC_H2D, [(crk.K_U64, b2), (crk.K_OPAQUE_VAR, ta), (crk.K_U64, ta.numel())], ring2, 0)
    cur += ctx.encode_call(2, gen.PROC_H2D, [(crk.K_U64, b2 + (1 << 20)), (crk.K_OPAQUE_VAR, tb), (crk.K_U64, tb.numel())],
                           ring2, cur)
    cur += ctx.encode_call(3, gen.PROC_D2H, [(crk.K_U64, b2 + (3 << 20)), (crk.K_U64, Cm.nbytes)], ring2, cur)
    send2 = crk.Ring.device(1 << 21)
    idx2 = ctx.index(1, 1024, 16)
    res.append(run("serve C2 matrixMul batch", ctx,
                   lambda: idx2.serve([(ring2, 0, cur)], [send2], [0], b2, region2.numel()), a.reps))
    # persistent server: phase-end markers of the last step (slot 6 = step start)
    L = crk.lib()
    tl = torch.zeros(16, dtype=torch.int64, device="cuda")
    L.crk_debug_timeline.restype = C.c_int
    L.crk_debug_timeline.argtypes = [C.c_void_p, C.c_void_p]
    for case, (ix_, rg, wn) in {"server 1 x 4 KiB HtoD": (ctx.index(1, 64, 16), ring, w),
                                "server C2 batch": (ctx.index(1, 1024, 16), ring2, cur)}.items():
        L.crk_debug_timeline(ctx.h, tl.data_ptr())
        torch.cuda.synchronize()
        srv = crk.Server(ix_, [rg], [send2], b2 if rg is ring2 else base, region2.numel() if rg is ring2 else region.numel())
        try:
            marks = []
            for _ in range(a.reps):
                tl.zero_()
                torch.cuda.current_stream().synchronize()
                out = srv.step([(0, wn)], [0])
                t = tl.cpu().numpy().reshape(8, 2)[:, 1]  # contiguous copy: no allocation while the server runs
                marks.append([int(t[i]) - int(t[6]) for i in (0, 1, 2, 3, 4, 5)] + [out["device_ns"]])
        finally:
            srv.stop()
            L.crk_debug_timeline(ctx.h, None)
        m = np.median(np.array(marks), axis=0) / 1e3
        res.append({"case": case, "after_setup_us": m[0], "after_scan_us": m[1], "after_parse_us": m[2],
                    "after_plan_us": m[3], "after_move_us": m[4], "after_publish_us": m[5], "device_us": m[6]})
    print(json.dumps(res))


if __name__ == "__main__":
    main()
