"""Per-round timing of the fragment scan (K1) on the bench workload, from the diagnostic build's clock
trace (build.py build_trace, -DCRK_SCAN_TRACE).  Prints, per mode (warp round / chase hop / CTA round),
how many and how long (SM cycles), and the slowest ring's total.

  python tools/scan_trace.py [--streams 16] [--payload-mib 64] [--host]
"""
import argparse
import collections
import ctypes as C
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_sc_eilingkkflm23_b200 import build  # noqa: E402

os.environ["CRK_LIB"] = build.build_trace()

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_sc_eilingkkflm23_b200 import crk, workload  # noqa: E402

MODES = {0: "end", 1: "warp_compute", 2: "chase", 3: "cta", 4: "warp_loads"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--streams", type=int, default=16)
    ap.add_argument("--payload-mib", type=int, default=64)
    ap.add_argument("--host", action="store_true")
    ap.add_argument("--touch", type=int, default=0, help="read one byte per TOUCH bytes of each ring first")
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    ctx = crk.Context(0)
    ep = workload.c5_endpoint(ctx, 0, dev, n_streams=a.streams, payload_per_stream=a.payload_mib << 20,
                              host_rings=a.host)
    idx = ctx.index(max_rings=a.streams, max_frags=1 << 20, max_records=1 << 14)
    L = crk.lib()
    L.crk_debug_scan_trace.argtypes = [C.c_void_p, C.c_void_p, C.c_int]
    buf = np.zeros((64, 4096), np.uint64)
    cnt = np.zeros(64, np.uint32)
    out = {}
    for rep in range(3):
        workload.serve_step(idx, ep)
        torch.cuda.synchronize()
        L.crk_debug_scan_trace(None, None, 1)
        if a.touch:
            for r, h, t in ep.rings:
                r.tensor()[::a.touch].sum()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        idx.frame_scan(ep.rings)
        e1.record()
        torch.cuda.synchronize()
        L.crk_debug_scan_trace(buf.ctypes.data, cnt.ctypes.data, 0)
        stats = collections.defaultdict(list)
        ring_tot = []
        for r in range(a.streams):
            n = int(cnt[r])
            e = buf[r, :n]
            clk = (e & ((1 << 40) - 1)).astype(np.int64)
            mode = (e >> 40) & 7
            hdr = e >> 43
            for i in range(1, n):
                stats[MODES[int(mode[i])]].append((int(clk[i] - clk[i - 1]), int(hdr[i])))
            ring_tot.append(int(clk[-1] - clk[0]) if n > 1 else 0)
        out = {"touch": a.touch, "scan_ms": round(e0.elapsed_time(e1), 4), "rings": a.streams,
               "slowest_ring_cycles": max(ring_tot), "mean_ring_cycles": int(np.mean(ring_tot)),
               "entries_per_ring": [int(c) for c in cnt[:a.streams]]}
        for m, v in stats.items():
            cyc = np.array([x[0] for x in v])
            out[m] = {"n": len(v), "mean_cycles": int(cyc.mean()), "p50": int(np.median(cyc)),
                      "p90": int(np.percentile(cyc, 90)), "headers": int(sum(x[1] for x in v))}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
