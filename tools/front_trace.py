"""Diagnostic: phase ends of the fused front end (build variant -DCRK_FRONT_TRACE) for smoke()'s two-record step
(12,345-byte HtoD in 4 KiB fragments + 10,000-byte DtoH): setup | scan | parse | plan, the first (cold) call
and the median of warm repeats."""
import ctypes as C
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle as O  # noqa: E402
from paper_conf_sc_eilingkkflm23_b200 import build, crk, gen  # noqa: E402

crk.LIBPATH = build.build_variant("ftrace", ["CRK_FRONT_TRACE"])
L = crk.lib()
L.crk_debug_front_trace.argtypes = [C.c_void_p]
F = 4096
cfg = O.Config(prog=gen.PROG, vers=gen.VERS, frag_payload=F)
ctx = crk.Context(0, frag_payload=F)
region = torch.zeros(1 << 16, dtype=torch.uint8, device="cuda")
base = region.data_ptr()
payload = gen.random_bytes(2, 12345)
wire = (O.encode_call(1, gen.PROC_H2D, [(O.K_U64, base + 3), (O.K_OPAQUE_VAR, payload.tobytes()),
                                        (O.K_U64, len(payload))], cfg)
        + O.encode_call(2, gen.PROC_D2H, [(O.K_U64, base + 30000), (O.K_U64, 10000)], cfg))
ring = crk.Ring.device(1 << 16)
ring.write(0, wire)
send = crk.Ring.device(1 << 16)
idx = ctx.index(1, 1024, 64)
out = []
for i in range(50):
    idx.serve([(ring, 0, len(wire))], [send], [0], base, region.numel())
    torch.cuda.synchronize()
    buf = np.zeros(8, np.uint64)
    L.crk_debug_front_trace(buf.ctypes.data)
    out.append(np.diff(buf[:5].astype(np.int64)) / 1e3)
names = ["setup", "scan", "parse", "plan"]
print("cold:", dict(zip(names, out[0].round(2).tolist())))
print("warm median:", dict(zip(names, np.median(np.array(out[5:]), axis=0).round(2).tolist())))
