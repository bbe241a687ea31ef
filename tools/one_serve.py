import sys, os
sys.path.insert(0, os.getcwd())
import torch
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
for i in range(60):
    idx.serve([(ring, 0, w)], [send], [0], base, region.numel())
torch.cuda.synchronize()
print("ok")
