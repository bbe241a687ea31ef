"""Diagnostic: sub-phase times of plan_small_block inside the persistent server (build variant with
-DCRK_PLAN_TRACE, made by build.build_variant) for one 4 KiB HtoD CALL per step: decide | stripe check + wire |
reply-offset scan | reply jobs | tile scans | clear + mover cursors.  The trace is read after each server stop
(a device-wide copy would wait for the running server)."""
import ctypes as C
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_eilingkkflm23_b200 import build, crk, gen  # noqa: E402

crk.LIBPATH = build.build_variant("ptrace", ["CRK_PLAN_TRACE"])
L = crk.lib()
L.crk_debug_server_plan_trace.argtypes = [C.c_void_p]
dev = torch.device("cuda:0")
ctx = crk.Context(0)
region = torch.zeros(1 << 22, dtype=torch.uint8, device=dev)
base = region.data_ptr()
data = torch.from_numpy(gen.random_bytes(0xC1, 4096)).to(dev)
ring = crk.Ring.device(1 << 14)
w = ctx.encode_call(7, gen.PROC_H2D, [(crk.K_U64, base + 4096), (crk.K_OPAQUE_VAR, data), (crk.K_U64, 4096)], ring, 0)
send = crk.Ring.device(1 << 16)
idx = ctx.index(1, 64, 16)
torch.cuda.synchronize()
d, phs = [], []
for rep in range(int(os.environ.get("REPS", "6"))):
    srv = crk.Server(idx, [ring], [send], base, region.numel())
    try:
        for i in range(20):
            out = srv.step([(0, w)], [0])
        phs.append(list(out["phase_end_ns"].values()))
    finally:
        srv.stop()
    buf = np.zeros(16, np.uint64)
    L.crk_debug_server_plan_trace(buf.ctypes.data)
    d.append(np.diff(buf[:7].astype(np.int64)) / 1e3)
    print("rep", rep, d[-1].round(2).tolist(), flush=True)
d = np.median(np.array(d), axis=0)
print("plan sub-phases (us, median):", dict(zip(["decide", "stripe+wire", "offset_scan", "reply_jobs", "tile_scans",
                                                   "clear+final"], d.round(2).tolist())))
print("server phase ends (ns):", np.median(np.array(phs), axis=0).tolist())
