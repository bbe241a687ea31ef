"""Sweeps library knobs on the bench workload (device-resident rings): per config, the step time and
the per-stage device times.  Usage: python tools/sweep.py 'tile_bytes=16384,mover_stages=4' ..."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sc_eilingkkflm23_b200 import build, crk, workload  # noqa: E402


def time_cfg(ep, kw, steps=50):
    ctx = crk.Context(0, **kw)
    idx = ctx.index(max_rings=len(ep.rings), max_frags=1 << 20, max_records=1 << 14)
    for _ in range(3):
        idx.serve(ep.rings, ep.sends, ep.offs, ep.base, ep.region.numel())
    torch.cuda.synchronize()
    crk.profile_enable(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps):
        idx.serve(ep.rings, ep.sends, ep.offs, ep.base, ep.region.numel())
    e1.record()
    torch.cuda.synchronize()
    prof = crk.profile_read()
    crk.profile_enable(False)
    ok = workload.check_results(idx, ep)["ok"]
    ms = e0.elapsed_time(e1) / steps
    return dict(cfg=kw, ms=round(ms, 4), gbs=round(ep.payload / ms / 1e6, 1), ok=ok,
                stages={k: round(v[0] / max(1, v[1]), 4) for k, v in prof.items()})


def main():
    build.build()
    base = crk.Context(0)
    ep = workload.c5_endpoint(base, 0, torch.device("cuda:0"))
    for arg in sys.argv[1:]:
        kw = {}
        for part in arg.split(","):
            if part:
                k, v = part.split("=")
                kw[k] = int(v, 0)
        try:
            print(json.dumps(time_cfg(ep, kw)), flush=True)
        except Exception as e:
            print(json.dumps(dict(cfg=kw, error=repr(e))), flush=True)


if __name__ == "__main__":
    main()
