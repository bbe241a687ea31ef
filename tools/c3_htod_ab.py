"""C3 HtoD (one memcpy CALL, crk_rpc_frame_scan + crk_xdr_decode_memcpy_h2d) per size under context variants, to
locate the fixed per-call cost of the launched path.  Device rings, buffers rotated over >= 256 MiB.

  python tools/c3_htod_ab.py [log2n,...] [variant,...]     variants: default, one_cta (scan_chunking=1), ...
Writes one JSON object (stdout)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import torch  # noqa: E402

import suite  # noqa: E402
from paper_conf_sc_eilingkkflm23_b200 import build, crk, gen  # noqa: E402

MiB = 1 << 20
VARIANTS = {"default": {}, "one_cta": {"scan_chunking": 1}}


def run(lg, kw):
    dev = suite.dev
    ctx = crk.Context(0, **kw)
    n = 1 << lg
    payload = torch.from_numpy(gen.c3_payload(lg)).to(dev)
    one = crk.Ring.device(suite.next_pow2(n + 4 * (n // 65536 + 2) + 64))
    w = ctx.encode_call(lg, gen.PROC_H2D, [(crk.K_U64, 0), (crk.K_OPAQUE_VAR, payload), (crk.K_U64, n)], one, 0)
    copies = max(1, min(64, (256 * MiB) // max(w, 1)))
    rings = [one] + [crk.Ring.device(one.cap) for _ in range(copies - 1)]
    for r in rings[1:]:
        r.tensor()[:w].copy_(one.tensor()[:w])
    dsts = [torch.empty(n, dtype=torch.uint8, device=dev) for _ in range(copies)]
    idx = ctx.index(1, n // 65536 + 16, 4)
    st = torch.zeros(1, dtype=torch.int32, device=dev)

    def scan(i):
        idx.frame_scan([(rings[i % copies], 0, w)])

    def h2d(i):
        scan(i)
        idx.decode_memcpy_h2d(lg, dsts[i % copies], n, st)

    reps = max(10, min(200, (1 << 30) // n))
    out = {"h2d_us": round(suite.timed(h2d, reps) * 1e3, 2), "scan_us": round(suite.timed(scan, reps) * 1e3, 2)}
    out["ok"] = bool(torch.equal(dsts[(reps - 1) % copies], payload)) and st.item() == 0
    out["scan_stats"] = idx.scan_stats()
    return out


def main():
    build.build()
    logs = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "12,20,22,24,26,28,30").split(",")]
    variants = (sys.argv[2] if len(sys.argv) > 2 else "default,one_cta").split(",")
    res = {}
    for v in variants:
        kw = VARIANTS[v] if v in VARIANTS else {k: int(x, 0) for k, x in (kv.split("=") for kv in v.split(";"))}
        res[v] = {lg: run(lg, kw) for lg in logs}
        torch.cuda.empty_cache()
    print(json.dumps(res))


if __name__ == "__main__":
    main()
