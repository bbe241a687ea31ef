"""GPU parity of striped memcpys (reading R22: Cricket's parallel-socket memcpy,
PAPER.md:170, :238, :240): memcpys split at random points into stripes sent over several rings, interleaved with
plain HtoD / DtoH calls, incomplete and inconsistent memcpys and failing stripes, served by crk_serve through
the one-block planner, the multi-kernel planner and the fused front end, and compared with the oracle's or_serve
on the same bytes: region, every send ring, every per-record status and reply discriminant."""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import crk, gen
from tests.gpu_util import ctx_for, d2h_call, h2d_call, make_ring, ocfg, ring_np

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("needs a GPU", allow_module_level=True)


def stripe_call(xid, ptr, data, offset, total, parent, size=None):
    return (xid, 3, [(O.K_U64, ptr), (O.K_OPAQUE_VAR, bytes(data)), (O.K_U64, len(data) if size is None else size),
                     (O.K_U32, parent), (O.K_U64, offset), (O.K_U64, total)])


def build(seed, base, region_bytes, n_rings, n_memcpy=6):
    g = gen.rng(seed)
    calls = [[] for _ in range(n_rings)]
    host_region = np.zeros(region_bytes, np.uint8)
    off, xid = 0, 1
    for m in range(n_memcpy):
        total = int(g.integers(1, 400_000))
        payload = gen.random_bytes(seed * 100 + m, total)
        k = int(g.integers(1, 2 * n_rings + 1))
        cuts = sorted(set(int(x) for x in g.integers(0, total, k - 1))) if k > 1 else []
        bounds = [0] + cuts + [total]
        parts = list(zip(bounds, bounds[1:]))
        drop = int(g.integers(0, len(parts))) if m == 4 else -1            # memcpy 4: a stripe never arrives
        for i in g.permutation(len(parts)).tolist():
            if i == drop:
                continue
            a, b = parts[i]
            t = total + (1 if (m == 5 and i == len(parts) - 1) else 0)     # memcpy 5: one stripe disagrees
            calls[int(g.integers(0, n_rings))].append(stripe_call(xid, base + off, payload[a:b], a, t, 0xAB00 + m))
            xid += 1
        off = (off + total + 255) // 256 * 256
    for r in range(n_rings):  # plain calls and failing stripes around them
        d = gen.random_bytes(seed + r, 5000)
        calls[r].insert(int(g.integers(0, len(calls[r]) + 1)), h2d_call(xid, d, base + off))
        host_region[off + 6000:off + 9000] = gen.random_bytes(seed + 77, 3000)
        calls[r].append(d2h_call(xid + 1, base + off + 6000, 3000))
        calls[r].append(stripe_call(xid + 2, base + off, d[:100], 50, 100, 0xEE00 + r))              # E_SIZE
        calls[r].append(stripe_call(xid + 3, base + region_bytes - 10, d[:100], 0, 100, 0xEF00 + r))  # E_PTR
        xid += 4
        off += 10_000
    assert off < region_bytes
    return calls, host_region


@pytest.mark.parametrize("path", ["small", "multi", "fused"])
@pytest.mark.parametrize("seed", [1, 2])
def test_striped_memcpys_match_oracle(path, seed):
    cfg = ocfg(F=16384)
    kw = {"small": {}, "multi": {}, "fused": {"fused_front_max_records": 1024, "fused_front_max_window": 1 << 40}}[path]
    ctx = ctx_for(cfg, **kw)
    n_rings = 4
    region_bytes = 4 << 20
    region = torch.zeros(region_bytes, dtype=torch.uint8, device="cuda")
    base = region.data_ptr()
    calls, host_region = build(seed, base, region_bytes, n_rings)
    region.copy_(torch.from_numpy(host_region))
    rings, sends, offs = [], [], []
    for r in range(n_rings):
        ring = make_ring(1 << 22)
        cur = 64 * r
        for c in calls[r]:
            w = O.encode_call(*c, cfg)
            ring.write(cur, w)
            cur += len(w)
        rings.append((ring, 64 * r, cur))
        sends.append(make_ring(1 << 20))
        offs.append(8 * r)
    max_records = 1 << 11 if path == "multi" else 1 << 10  # above kSmallServe: the multi-kernel planner
    idx = ctx.index(n_rings, 1 << 14, max_records)
    for _ in range(2):  # twice: the parent table must be empty again for the second step
        idx.serve(rings, sends, offs, base, region_bytes)
    torch.cuda.synchronize()
    want = O.serve([(ring_np(r), h, t) for r, h, t in rings], cfg, host_region, base, [1 << 20] * n_rings, offs,
                   max_frags_per_ring=(1 << 14) // n_rings, max_records_per_ring=max_records // n_rings)
    T = idx.tables(n_rings)
    assert [r["status"] for r in want["records"]] == list(T["parsed"]["serve_status"])
    assert [r["reply_err"] for r in want["records"]] == list(T["parsed"]["serve_reply_err"])
    n_leads = sum(1 for r in want["records"] if r["proc"] == 3 and r["reply_err"] == 0)
    assert n_leads == 4  # memcpys 0-3 complete; 4 (a stripe missing) and 5 (inconsistent) do not
    assert np.array_equal(region.cpu().numpy(), host_region)
    for r in range(n_rings):
        n = want["reply_bytes"][r]
        assert T["rings"][r]["reply_bytes"] == n
        assert sends[r].read(offs[r], n) == bytes(want["send"][r][offs[r]:offs[r] + n])
