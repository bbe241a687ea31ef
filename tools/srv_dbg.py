import sys, os, time
sys.path.insert(0, os.getcwd())
if len(sys.argv) > 1:
    from paper_conf_sc_eilingkkflm23_b200 import build
    os.environ["CRK_LIB"] = build.build_variant("timeline2", ["CRK_TIMELINE", "CRK_TIMELINE_SCAN2"])
import ctypes as C
import numpy as np, torch
from paper_conf_sc_eilingkkflm23_b200 import crk, gen
dev = torch.device("cuda:0")
ctx = crk.Context(0)
region = torch.zeros(1 << 20, dtype=torch.uint8, device=dev)
base = region.data_ptr()
data = torch.from_numpy(gen.random_bytes(0xC1, 4096)).to(dev)
ring = crk.Ring.device(1 << 14)
w = ctx.encode_call(7, gen.PROC_H2D, [(crk.K_U64, base + 4096), (crk.K_OPAQUE_VAR, data), (crk.K_U64, 4096)], ring, 0)
send = crk.Ring.device(1 << 12)
idx = ctx.index(1, 64, 16)
tl = torch.zeros(16, dtype=torch.int64, device="cuda")
if len(sys.argv) > 1:
    L = crk.lib(); L.crk_debug_timeline.restype = C.c_int; L.crk_debug_timeline.argtypes = [C.c_void_p, C.c_void_p]
    L.crk_debug_timeline(ctx.h, tl.data_ptr())
torch.cuda.synchronize()
print("start", flush=True)
srv = crk.Server(idx, [ring], [send], base, region.numel())
print("started", flush=True)
try:
    for i in range(int(os.environ.get("STEPS", "5"))):
        out = srv.step([(0, w)], [0], timeout_s=5)
        t = tl.cpu().numpy().reshape(8, 2)[:, 1]
        print(i, out["status"], out["device_ns"], [int(t[k]) - int(t[6]) for k in (0, 1, 7, 2, 3, 4, 5)], flush=True)
        tl.zero_()
        torch.cuda.current_stream().synchronize()
        print("zeroed", tl.cpu().numpy()[12:14], flush=True)
finally:
    print("stopping", flush=True)
    srv.stop()
print("done", flush=True)
