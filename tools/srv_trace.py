"""Clock trace of the persistent server's scan phase (diagnostic build -DCRK_SCAN_TRACE)."""
import ctypes as C, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_eilingkkflm23_b200 import build
os.environ["CRK_LIB"] = build.build_variant("strace", ["CRK_SCAN_TRACE"])
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
L = crk.lib()
f = L.crk_debug_server_scan_trace
f.restype = C.c_int
f.argtypes = [C.c_void_p, C.c_void_p, C.c_int]
buf = np.zeros((64, 4096), np.uint64)
cnt = np.zeros(64, np.uint32)
f(None, None, 1)
torch.cuda.synchronize()
srv = crk.Server(idx, [ring], [send], base, region.numel())
try:
    for i in range(4):
        out = srv.step([(0, w)], [0])
    print("device_ns", out["device_ns"], flush=True)
finally:
    srv.stop()
torch.cuda.synchronize()
f(buf.ctypes.data, cnt.ctypes.data, 0)
n = int(cnt[0])
e = buf[0, :n]
clk = (e & ((1 << 40) - 1)).astype(np.int64)
mode = (e >> 40) & 7
hdr = e >> 43
names = {0: "end", 1: "warp_compute", 2: "chase", 3: "cta", 4: "warp_loads", 5: "scan_start"}
for k in range(n):
    print(k, names.get(int(mode[k])), int(hdr[k]), int(clk[k] - clk[k - 1]) if k else 0)
