"""Diagnostic: the persistent server's step trace (build variant with -DCRK_STEP_TRACE, made by
build.build_variant) for one 4 KiB HtoD CALL per step: %globaltimer at numbered points (crk_device.cuh
STEP_MARK), each taken once the value it depends on has arrived.  Points: 0 scan start; 8-13 inside
parse_record (entry, record table, fragment table, ring bytes, lane-0 checks, tables written); 16 jobs staged;
17 tiles moved; 18 after the move barrier; 19 results published; 20 done_seq released.  Lean steps: 21 windows
copied, 22 walked, 23 checked, 24 offsets, 25 decided, 1 ring results and 2 record rows written, 26 tables done,
27-30 first warps' moves, 31 replies encoded.  The trace is read
after each server stop (a device-wide copy would wait for the running server)."""
import ctypes as C
import zlib
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_eilingkkflm23_b200 import build, crk, gen  # noqa: E402

VARIANT = os.environ.get("VARIANT", "")  # extra -D defines, ';'-separated, e.g. an inlining experiment
O3 = os.environ.get("ALL_O3") == "1"  # every file at the default flags (no build.FILE_FLAGS)
crk.LIBPATH = build.build_variant("steptrace" + (f"{zlib.crc32(VARIANT.encode()):08x}" if VARIANT else "") +
                                  ("_o3" if O3 else ""), ["CRK_STEP_TRACE"] + [d for d in VARIANT.split(";") if d],
                                  file_flags={} if O3 else None)
L = crk.lib()
L.crk_debug_server_step_trace.argtypes = [C.c_void_p]
dev = torch.device("cuda:0")
ctx = crk.Context(0)
region = torch.zeros(1 << 22, dtype=torch.uint8, device=dev)
base = region.data_ptr()
data = torch.from_numpy(gen.random_bytes(0xC1, 4096)).to(dev)
ring = crk.Ring.device(1 << 16)
w = 0
if os.environ.get("CONTROL") == "1":  # one control call of a registered procedure instead (suite.py's)
    ctx.register_schema(60, [crk.K_U64, crk.K_U32, crk.K_U32, crk.K_OPAQUE_VAR])
    w = ctx.encode_call(9, 60, [(crk.K_U64, 0x7F00DEADBEEF), (crk.K_U32, 148), (crk.K_U32, 256),
                                (crk.K_OPAQUE_VAR, data[:64])], ring, 0)
for i in range(0 if w else int(os.environ.get("CALLS", "1"))):  # CALLS=12: a step of twelve 4 KiB HtoD calls
    w += ctx.encode_call(7 + i, gen.PROC_H2D, [(crk.K_U64, base + 4096 * (i + 1)), (crk.K_OPAQUE_VAR, data),
                                              (crk.K_U64, 4096)], ring, w)
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
    buf = np.zeros(32, np.uint64)
    L.crk_debug_server_step_trace(buf.ctypes.data)
    pts = [i for i in range(32) if buf[i]]
    t0 = int(buf[0])
    d.append([(int(buf[i]) - t0) / 1e3 for i in pts])
    print("rep", rep, dict(zip(pts, np.round(d[-1], 2).tolist())), flush=True)
d = np.median(np.array(d), axis=0)
print("step points (us after scan start, median):", dict(zip(pts, d.round(2).tolist())))
print("server phase ends (ns):", np.median(np.array(phs), axis=0).tolist())
