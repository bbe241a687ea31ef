"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py times (default context).

* C3 1 GiB HtoD record (16,385 fragments): fragment table == oracle, dst == payload (decode(encode(x)) = x
  with the oracle's encoder), closed-form wire size.
* C3 1 GiB DtoH reply: every byte == the oracle's encoding.
* C5 full endpoint (16 streams x 64 MiB, the bench workload) with oracle-encoded rings: region, send rings,
  per-record statuses and per-ring results == oracle or_serve.
* C1 x 131,072 back-to-back single-fragment records: scan/parse == oracle on a sample; typed + opaque
  decode of sampled records.
* C4 256 MiB typed-array stress, regular and irregular framing: every item == the generator's values.
"""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import crk, gen
from tests.gpu_util import compare_scan, ocfg

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("needs a GPU", allow_module_level=True)

GiB, MiB = 1 << 30, 1 << 20


def dev_ring_from(wire: np.ndarray, cap: int, at: int = 0) -> crk.Ring:
    r = crk.Ring.device(cap)
    t = torch.from_numpy(wire)
    n = len(wire)
    first = min(n, cap - at)
    r.tensor()[at:at + first].copy_(t[:first])
    if first < n:
        r.tensor()[:n - first].copy_(t[first:])
    return r


def test_c3_1gib_htod_decode():
    cfg = ocfg()
    ctx = crk.Context(0)
    payload = gen.c3_payload(30)
    L = O.call_header(0xC3, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0x1000) + O.put_u32(len(payload))
    wire = np.frombuffer(O.frame(L + payload.tobytes() + O.put_u64(len(payload)), 65536), np.uint8)
    assert len(wire) == 1_073_807_424 == O.wire_size(GiB + 60, 65536)
    at = (1 << 31) - 777
    ring = dev_ring_from(wire, 1 << 31, at)
    idx = ctx.index(1, 1 << 15, 16)
    idx.frame_scan([(ring, at, at + len(wire))])
    T = idx.tables()
    assert T["frags"][0]["hdr"].shape[0] == 16385
    # oracle scan on the same bytes (host copy of the ring window)
    ring_host = np.zeros(1 << 31, np.uint8)
    ring_host[at:] = wire[:(1 << 31) - at]
    ring_host[:len(wire) - ((1 << 31) - at)] = wire[(1 << 31) - at:]
    compare_scan(T, 0, ring_host, at, at + len(wire), 1 << 15, 16)
    del ring_host
    dst = torch.empty(GiB, dtype=torch.uint8, device="cuda")
    st = torch.zeros(1, dtype=torch.int32, device="cuda")
    cp = torch.zeros(1, dtype=torch.int64, device="cuda")
    idx.decode_memcpy_h2d(0xC3, dst, GiB, st, cp)
    torch.cuda.synchronize()
    assert st.item() == O.OK and cp.item() == GiB
    assert torch.equal(dst, torch.from_numpy(payload).cuda())


def test_c3_1gib_dtoh_encode():
    ctx = crk.Context(0)
    payload = gen.c3_payload(30)
    src = torch.from_numpy(payload).cuda()
    out = crk.Ring.device(1 << 31)
    at = (1 << 31) - 12345
    w = ctx.encode_memcpy_d2h(0xD3, src, 0, out, at)
    want = np.frombuffer(O.encode_memcpy_d2h(0xD3, payload, 0, 65536), np.uint8)
    assert w == len(want) == 1_073_807_396
    torch.cuda.synchronize()
    t = out.tensor()
    got = torch.cat([t[at:], t[:w - ((1 << 31) - at)]])
    assert torch.equal(got, torch.from_numpy(want).cuda())


def test_c5_full_endpoint_serve_matches_oracle():
    cfg = ocfg()
    ctx = crk.Context(0)
    streams, region_bytes = gen.c5_endpoint(0, n_streams=16, payload_per_stream=64 * MiB,
                                            h2d_budget=60 * MiB)
    region = torch.zeros(region_bytes + 256, dtype=torch.uint8, device="cuda")
    base = region.data_ptr()
    host_region = np.zeros(region_bytes + 256, np.uint8)
    rings, ring_np, sends, offs = [], [], [], []
    for s in streams:
        wires = []
        for r in s.records:
            d = gen.random_bytes(r.seed & 0xFFFFFFFF, r.size)
            if r.kind == gen.PROC_H2D:
                wires.append(O.encode_call(r.xid, r.kind, [(O.K_U64, base + r.region_off), (O.K_OPAQUE_VAR, d),
                                                           (O.K_U64, r.size)], cfg))
            else:
                host_region[r.region_off:r.region_off + r.size] = d
                wires.append(O.encode_call(r.xid, r.kind, [(O.K_U64, base + r.region_off), (O.K_U64, r.size)], cfg))
        w = np.frombuffer(b"".join(wires), np.uint8)
        cap = 1 << 26
        assert len(w) <= cap
        hb = np.zeros(cap, np.uint8)
        hb[:len(w)] = w
        ring_np.append((hb, 0, len(w)))
        rings.append((dev_ring_from(w, cap), 0, len(w)))
        sends.append(crk.Ring.device(1 << 27))
        offs.append(64 * s.stream)
    region.copy_(torch.from_numpy(host_region))
    idx = ctx.index(16, 1 << 20, 1 << 14)
    idx.serve(rings, sends, offs, base, region.numel())
    torch.cuda.synchronize()
    T = idx.tables(16)
    want = O.serve(ring_np, cfg, host_region, base, [1 << 27] * 16, offs, max_frags_per_ring=(1 << 20) // 16,
                   max_records_per_ring=(1 << 14) // 16)
    assert all(s == O.OK for s in want["scan_status"])
    assert [r["status"] for r in want["records"]] == list(T["parsed"]["serve_status"])
    assert all(r["status"] == O.OK for r in want["records"])
    assert torch.equal(region, torch.from_numpy(host_region).cuda())
    for r in range(16):
        g = T["rings"][r]
        assert g["consumed"] == want["consumed"][r] and g["reply_bytes"] == want["reply_bytes"][r]
        n = want["reply_bytes"][r]
        got = sends[r].tensor()[offs[r]:offs[r] + n]
        assert torch.equal(got, torch.from_numpy(want["send"][r][offs[r]:offs[r] + n]).cuda())


def test_c1_back_to_back_records():
    cfg = ocfg(user={gen.PROC_C1: gen.C1_SCHEMA})
    ctx = crk.Context(0)
    ctx.register_schema(gen.PROC_C1, gen.C1_SCHEMA)
    n = 131072
    c1 = gen.c1_call(xid=0)
    one = O.encode_call(0, c1.proc, [(k, v.tobytes() if k == O.K_OPAQUE_VAR else v) for k, v in c1.items], cfg)
    assert len(one) == 8260
    wire = np.tile(np.frombuffer(one, np.uint8), n)
    xids = np.arange(n, dtype=np.uint32) + 0x10000
    wire.reshape(n, 8260)[:, 4:8] = xids.astype(">u4").view(np.uint8).reshape(n, 4)  # xid word of each CALL
    ring = dev_ring_from(wire, 1 << 31)
    idx = ctx.index(1, 1 << 18, 1 << 18)
    idx.frame_scan([(ring, 0, len(wire))])
    T = idx.tables()
    assert T["rings"][0]["status"] == O.OK and T["rings"][0]["n_records"] == n
    assert np.array_equal(T["parsed"]["xid"], xids)
    assert (T["parsed"]["status"] == O.OK).all()
    sample = np.random.default_rng(1).choice(n, 64, replace=False)
    s = O.frame_scan(wire[:8260 * 3], 0, 8260 * 3)
    for d in sample:
        assert T["recs"][0]["begin"][d] == 8260 * d and T["recs"][0]["len"][d] == 8256
        assert T["parsed"]["count"][d, 3] == 1024 and T["parsed"]["off"][d, 3] == 4160
    outs = torch.zeros((len(sample), 1024), dtype=torch.int32, device="cuda")
    cnt = torch.zeros(len(sample), dtype=torch.int64, device="cuda")
    st = torch.zeros(len(sample), dtype=torch.int32, device="cuda")
    reqs = [(int(xids[d]), 3, O.K_I32_VAR, outs[i].data_ptr(), 1024, cnt.data_ptr() + 8 * i, st.data_ptr() + 4 * i)
            for i, d in enumerate(sample)]
    keep = idx.decode_items_batch(reqs)
    torch.cuda.synchronize()
    assert (st.cpu().numpy() == O.OK).all() and (cnt.cpu().numpy() == 1024).all()
    want = torch.from_numpy(c1.items[3][1]).cuda()
    assert all(torch.equal(outs[i], want) for i in range(len(sample)))
    del keep


@pytest.mark.parametrize("irregular", [False, True])
def test_c4_typed_stress_256mib(irregular):
    cfg = ocfg(user=gen.C4_SCHEMAS)
    ctx = crk.Context(0)
    for proc, items in gen.C4_SCHEMAS.items():
        ctx.register_schema(proc, items)
    calls = gen.c4_calls(256 * MiB)
    wires = []
    for c in calls:
        L = O.call_header(c.xid, gen.PROG, gen.VERS, c.proc) + b"".join(
            O.encode_item(k & 0xFF, v.tobytes() if (k & 0xFF) in (O.K_OPAQUE_VAR, O.K_OPAQUE_FIX) else v)
            for k, v in c.items)
        wires.append(O.frame_lens(L, gen.split_points(gen.frag_seed(c), len(L))) if irregular else O.frame(L, 65536))
    wire = np.frombuffer(b"".join(wires), np.uint8)
    ring = dev_ring_from(wire, 1 << 29)
    idx = ctx.index(1, 1 << 16, 1 << 12)
    idx.frame_scan([(ring, 0, len(wire))])
    T = idx.tables()
    assert T["rings"][0]["status"] == O.OK and T["rings"][0]["n_records"] == len(calls)
    assert (T["parsed"]["status"] == O.OK).all()
    reqs, outs, want = [], [], []
    st = torch.full((4096,), 99, dtype=torch.int32, device="cuda")
    for c in calls:
        for a, (code, v) in enumerate(c.items):
            k = code & 0xFF
            if k in (O.K_U32, O.K_U64):
                continue
            raw = v.view(np.uint8) if k not in (O.K_OPAQUE_VAR, O.K_OPAQUE_FIX) else v
            out = torch.empty(len(raw) + 16, dtype=torch.uint8, device="cuda")
            reqs.append((c.xid, a, k, out.data_ptr(), len(v), None, st.data_ptr() + 4 * len(reqs)))
            outs.append(out)
            want.append(raw)
    keep = idx.decode_items_batch(reqs)
    torch.cuda.synchronize()
    assert (st[:len(reqs)].cpu().numpy() == O.OK).all()
    for out, w in zip(outs, want):
        assert torch.equal(out[:len(w)], torch.from_numpy(np.ascontiguousarray(w)).cuda())
    del keep
