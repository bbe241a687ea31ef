"""Diagnostic: the lean-boundary fuzz's clean trials through the persistent server (build variant with
-DCRK_LEAN_WHY): per trial, whether the lean path took the step and, when not, the reason word it left in the bell."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle as O  # noqa: E402
from paper_conf_sc_eilingkkflm23_b200 import build, crk, gen  # noqa: E402
from tests.gpu_util import ctx_for, make_ring, ocfg  # noqa: E402
from tests.test_gpu_fuzz import stream  # noqa: E402

crk.LIBPATH = build.build_variant("leanwhy", ["CRK_LEAN_WHY"])
cfg = ocfg(strict=True, F=1024, user={40: [O.K_U32, O.K_OPAQUE_VAR]})
ctx = ctx_for(cfg, max_record_bytes=1 << 14, lean_backoff=0)
region = torch.zeros(1 << 17, dtype=torch.uint8, device="cuda")
base = region.data_ptr()
g = gen.rng(99)
idx = ctx.index(4, 1 << 12, 256)
cap, scap = 1 << 16, 1 << 17
rings = [make_ring(cap) for _ in range(4)]
sends = [make_ring(scap) for _ in range(4)]
tails = [0, 0, 0, 0]
offs = [0, 0, 0, 0]
torch.cuda.synchronize()
srv = crk.Server(idx, rings, sends, base, region.numel())
try:
    for trial in range(12):
        heads = list(tails)
        for r in range(4):
            w = stream(g, cfg, base, int(g.choice([64, 256, 1024, 1 << 16])), 8 * r, distinct=True)
            wire = b"".join(bytes(x) for x in w)
            rings[r].write(heads[r], wire)
            tails[r] = heads[r] + len(wire)
        torch.cuda.current_stream().synchronize()
        out = srv.step(list(zip(heads, tails)), offs)
        ph = list(out["phase_end_ns"].values())
        why = srv.bell.pad_
        print(trial, "lean" if ph[1] == ph[2] == ph[3] == ph[4] else "general", "why", hex(why),
              "walk_ok", why & 1, "d2h_over", (why >> 1) & 1, "nrec", (why >> 2) & 0x3fff, "bad", hex(why >> 16),
              [r["status"] for r in out["results"]], flush=True)
        for r in range(4):
            tails[r] = out["results"][r]["consumed"]
            offs[r] += out["results"][r]["reply_bytes"]
finally:
    srv.stop()
