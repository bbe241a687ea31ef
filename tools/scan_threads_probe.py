"""Frame-scan latency of one small record vs the scan CTA size (diagnostic)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_eilingkkflm23_b200 import crk, gen
dev = torch.device("cuda:0")
for th in (64, 128, 256, 512, 1024):
    ctx = crk.Context(0, scan_threads=th)
    region = torch.zeros(1 << 20, dtype=torch.uint8, device=dev)
    data = torch.from_numpy(gen.random_bytes(0xC1, 4096)).to(dev)
    ring = crk.Ring.device(1 << 14)
    w = ctx.encode_call(7, gen.PROC_H2D, [(crk.K_U64, region.data_ptr()), (crk.K_OPAQUE_VAR, data), (crk.K_U64, 4096)], ring, 0)
    idx = ctx.index(1, 64, 16)
    for _ in range(20):
        idx.frame_scan([(ring, 0, w)])
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(200):
        idx.frame_scan([(ring, 0, w)])
    e1.record()
    torch.cuda.synchronize()
    print(th, round(e0.elapsed_time(e1) / 200 * 1e3, 2), "us per scan+parse", flush=True)
