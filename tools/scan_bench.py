"""K1 timing on the long-window configs (CUDA events, warm, device rings): C3 1 GiB HtoD record (16,385
fragments), C4-ii irregular 256 MiB stream, C5 endpoint (16 rings x 64 MiB).  SCAN_CFG picks configs,
SCAN_REPS the repetitions; SCAN_CTX crk_config overrides (e.g. scan_chunking=1).  Used under ncu for the K1
captures in profiles/."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle as O  # noqa: E402
from paper_conf_sc_eilingkkflm23_b200 import build, crk, gen, workload  # noqa: E402

MiB = 1 << 20
build.build()
KW = {k: int(v, 0) for k, v in (kv.split("=") for kv in os.environ.get("SCAN_CTX", "").split(",") if kv)}
REPS = int(os.environ.get("SCAN_REPS", "20"))
dev = torch.device("cuda:0")


def c3():
    n = 1 << 30
    payload = gen.c3_payload(30)
    L = O.call_header(0xC3, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0) + O.put_u32(n)
    w = np.frombuffer(O.frame(L + payload.tobytes() + O.put_u64(n), 65536), np.uint8)
    ring = crk.Ring.device(1 << 31)
    ring.tensor()[:len(w)].copy_(torch.from_numpy(w.copy()))
    return [(ring, 0, len(w))], (1, 1 << 15, 16)


def c4():
    cfg = O.Config(prog=gen.PROG, vers=gen.VERS)
    g = gen.rng(0xC4)
    parts, n, i = [], 0, 0
    while n < 256 * MiB:
        d = gen.random_bytes(i, gen.log_uniform_int(g, 1, 1 << 20))
        Lr = O.call_header(i, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0) + O.put_opaque_var(d.tobytes()) + \
            O.put_u64(len(d))
        parts.append(O.frame_lens(Lr, gen.split_points(gen.rng(i).integers(1 << 30), len(Lr))))
        n += len(parts[-1])
        i += 1
    w = np.frombuffer(b"".join(parts), np.uint8)
    ring = crk.Ring.device(1 << 29)
    ring.tensor()[:len(w)].copy_(torch.from_numpy(w.copy()))
    return [(ring, 0, len(w))], (1, 1 << 16, 1 << 12)


def c5():
    ctx = crk.Context(0)
    ep = workload.c5_endpoint(ctx, 0, dev)
    c5.keep = ep
    return ep.rings, (16, 1 << 20, 1 << 14)


out = {}
ctx = crk.Context(0, **KW)
for name in os.environ.get("SCAN_CFG", "c3,c4,c5").split(","):
    rings, shape = {"c3": c3, "c4": c4, "c5": c5}[name]()
    idx = ctx.index(*shape)
    for _ in range(3):
        idx.frame_scan(rings)
    torch.cuda.synchronize()
    crk.profile_enable(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(REPS):
        idx.frame_scan(rings)
    e1.record()
    torch.cuda.synchronize()
    prof = crk.profile_read()
    crk.profile_enable(False)
    res = idx.ring_results(len(rings))
    out[name] = {"frame_scan_us": round(e0.elapsed_time(e1) / REPS * 1e3, 2),
                 "stage_us": {k: round(v[0] / max(1, v[1]) * 1e3, 2) for k, v in prof.items() if v[1]},
                 "frags": sum(r["n_frags"] for r in res), "records": sum(r["n_records"] for r in res),
                 "ok": all(r["status"] == 0 for r in res), "scan_stats": idx.scan_stats(),
                 "window_bytes": sum(t - h for _, h, t in rings)}
    del idx, rings
    torch.cuda.empty_cache()
print(json.dumps(out))
