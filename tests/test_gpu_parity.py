"""GPU parity: the CUDA path (through the C ABI) against the oracle, bit-exact, on seeded inputs.

Sizes are small enough for the oracle to finish in seconds yet span many 16-byte chunks, several mover
tiles, fragment boundaries at every alignment and ragged tails.  Full-size checks live in
test_gpu_fullsize.py."""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import crk, gen
from tests.gpu_util import (compare_parse, compare_scan, ctx_for, d2h_call, h2d_call, make_ring, ocfg, ring_np)

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("needs a GPU", allow_module_level=True)


def place(ring, wire: bytes, head: int):
    ring.write(head, wire)
    return head + len(wire)


def mixed_stream(seed: int, n: int, cfg: O.Config, Fs=(64, 1000, 4096, 65536)):
    g = gen.rng(seed)
    wires, calls = [], []
    for i in range(n):
        kind = g.integers(0, 4)
        F = int(g.choice(Fs))
        if kind == 0:
            size = int(g.integers(0, 70000))
            c = h2d_call(1000 + i, gen.random_bytes(seed * 7919 + i, size))
        elif kind == 1:
            c = d2h_call(1000 + i, 0x7F0000000000 + int(g.integers(0, 1 << 20)), int(g.integers(0, 1 << 20)))
        elif kind == 2:
            c1 = gen.c1_call(xid=1000 + i)
            c = (c1.xid, c1.proc, [(k, v.tobytes() if k == O.K_OPAQUE_VAR else v) for k, v in c1.items])
        else:
            size = int(g.integers(1, 3000))
            c = h2d_call(1000 + i, gen.random_bytes(seed + i, size))
            F = int(g.integers(1, 200))
        w = O.encode_call(c[0], c[1], c[2], cfg, F=F)
        wires.append(w)
        calls.append(c)
    return wires, calls


@pytest.mark.parametrize("host", [False, True])
@pytest.mark.parametrize("at", [0, (1 << 20) - 37])
def test_scan_and_parse_match_oracle(host, at):
    cfg = ocfg(user={gen.PROC_C1: gen.C1_SCHEMA})
    ctx = ctx_for(cfg)
    wires, _ = mixed_stream(11, 60, cfg)
    cap = 1 << 21
    ring = make_ring(cap, host)
    tail = at
    for w in wires:
        tail = place(ring, w, tail)
    idx = ctx.index(max_rings=1, max_frags=1 << 14, max_records=1 << 10)
    idx.frame_scan([(ring, at, tail)])
    T = idx.tables()
    rb = ring_np(ring)
    s = compare_scan(T, 0, rb, at, tail, 1 << 14, 1 << 10)
    assert s.status == O.OK and len(s.recs) == 60
    compare_parse(T, 0, rb, s, cfg)


def test_scan_every_truncation():
    cfg = ocfg()
    ctx = ctx_for(cfg)
    wires, _ = mixed_stream(5, 4, cfg, Fs=(16, 40))
    ring = make_ring(1 << 16)
    tail = 0
    for w in wires:
        tail = place(ring, w, tail)
    rb = ring_np(ring)
    idx = ctx.index(1, 4096, 256)
    for t in list(range(0, min(tail, 400))) + list(range(max(0, tail - 200), tail + 1)):
        idx.frame_scan([(ring, 0, t)])
        T = idx.tables()
        compare_scan(T, 0, rb, 0, t, 4096, 256)


def test_scan_irregular_zero_fragments_and_regular_runs():
    cfg = ocfg(user={33: [O.K_U32]})
    ctx = ctx_for(cfg)
    g = gen.rng(77)
    ring = make_ring(1 << 22)
    tail = 5
    for i in range(40):
        L = O.call_header(i, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0) + \
            O.put_opaque_var(gen.random_bytes(i, int(g.integers(0, 20000))).tobytes())
        L += O.put_u64(len(L) - 52)
        lens = gen.split_points(i, len(L), 1, int(g.choice([3, 50, 7000])))
        # sprinkle zero-length fragments (reading R1) and sometimes an empty last one (R2)
        for _ in range(int(g.integers(0, 3))):
            lens.insert(int(g.integers(0, len(lens) + 1)), 0)
        if g.random() < 0.3:
            lens.append(0)
        tail = place(ring, O.frame_lens(L, lens), tail)
    # 300 identical single-fragment records (stride speculation across records)
    for i in range(300):
        tail = place(ring, O.encode_call(5000 + i, 33, [(O.K_U32, i)], cfg), tail)
    idx = ctx.index(1, 1 << 21, 1 << 11)
    idx.frame_scan([(ring, 5, tail)])
    T = idx.tables()
    rb = ring_np(ring)
    s = compare_scan(T, 0, rb, 5, tail, 1 << 21, 1 << 11)
    assert len(s.recs) == 340
    compare_parse(T, 0, rb, s, cfg)


@pytest.mark.parametrize("host", [False, True])
def test_scan_chase_irregular_long_chains(host):
    """Long runs of irregular fragment lengths (the scan's serial chase pass), interleaved with regular
    runs (hand-back to the speculative rounds), across the ring wrap; then every stop inside a chase:
    truncated windows, E_FRAG, fragment and record capacity."""
    cfg = ocfg()
    ctx = ctx_for(cfg)
    g = gen.rng(4242)
    cap = 1 << 22
    ring = make_ring(cap, host)
    head = cap - 300000
    tail = head
    for i in range(60):
        L = O.call_header(i, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0) + \
            O.put_opaque_var(gen.random_bytes(i, int(g.integers(0, 30000))).tobytes())
        L += O.put_u64(len(L) - 52)
        if i % 10 == 9:  # regular run: the speculative rounds take over again
            lens = [64] * (len(L) // 64) + [len(L) % 64]
        else:  # irregular, zero-length fragments included
            lens = gen.split_points(1000 + i, len(L), 0, int(g.choice([8, 300, 4000])))
        tail = place(ring, O.frame_lens(L, lens), tail)
    rb = ring_np(ring)
    idx = ctx.index(1, 1 << 20, 1 << 10)
    idx.frame_scan([(ring, head, tail)])
    s = compare_scan(idx.tables(), 0, rb, head, tail, 1 << 20, 1 << 10)
    assert len(s.recs) == 60 and len(s.frags) > 20000
    compare_parse(idx.tables(), 0, rb, s, cfg)
    frag_ends = [f["phys"] + f["len"] for f in s.frags]
    for t in [head + 3, frag_ends[5000] - 1, frag_ends[5000] + 2, frag_ends[12345], tail - 1]:
        idx.frame_scan([(ring, head, t)])
        compare_scan(idx.tables(), 0, rb, head, t, 1 << 20, 1 << 10)
    for fpr, rpr, mrb in [(7000, 1 << 10, 1 << 32), (1 << 20, 13, 1 << 32), (1 << 20, 1 << 10, 20000)]:
        c3 = crk.Context(0, frag_payload=65536, strict=1, prog=cfg.prog, vers=cfg.vers, max_record_bytes=mrb)
        i3 = c3.index(1, fpr, rpr)
        i3.frame_scan([(ring, head, tail)])
        compare_scan(i3.tables(), 0, rb, head, tail, fpr, rpr, mrb)


def test_scan_limits_frag_capacity_records():
    cfg = ocfg()
    ctx = ctx_for(cfg)
    wires, _ = mixed_stream(3, 12, cfg, Fs=(100, 500))
    ring = make_ring(1 << 21)
    tail = 0
    for w in wires:
        tail = place(ring, w, tail)
    rb = ring_np(ring)
    for fpr, rpr, mrb in [(1 << 14, 1 << 10, 1000), (1 << 14, 1 << 10, 5000), (7, 64, 1 << 32),
                          (200, 64, 1 << 32), (1 << 14, 3, 1 << 32), (1 << 14, 1, 1 << 32), (1, 1, 1 << 32)]:
        c3 = crk.Context(0, frag_payload=65536, strict=1, prog=cfg.prog, vers=cfg.vers, max_record_bytes=mrb)
        idx = c3.index(1, fpr, rpr)
        idx.frame_scan([(ring, 0, tail)])
        T = idx.tables()
        compare_scan(T, 0, rb, 0, tail, fpr, rpr, mrb)


def test_multi_ring_scan_dense_numbering_and_xid_dups():
    cfg = ocfg()
    ctx = ctx_for(cfg)
    rings, spec = [], []
    for r in range(5):
        ring = make_ring(1 << 18, host=(r % 2 == 1))
        wires, _ = mixed_stream(100 + r, 0 if r == 2 else 7 + r, cfg)
        tail = 64 * r
        for w in wires:
            tail = place(ring, w, tail)
        rings.append((ring, 64 * r, tail))
    idx = ctx.index(8, 1 << 15, 1 << 10)
    idx.frame_scan(rings)
    T = idx.tables(5)
    base = 0
    for r, (ring, h, t) in enumerate(rings):
        rb = ring_np(ring)
        s = compare_scan(T, r, rb, h, t, (1 << 15) // 8, (1 << 10) // 8)
        assert T["rings"][r]["rec_base"] == base
        compare_parse(T, r, rb, s, cfg)
        base += len(s.recs)
    assert T["total"] == base


def dst_buffer(nbytes: int, misalign: int, guard: int = 64):
    buf = torch.full((nbytes + 2 * guard + 16,), 0xA5, dtype=torch.uint8, device="cuda")
    return buf, buf.data_ptr() + guard + misalign


@pytest.mark.parametrize("size", [0, 1, 3, 15, 16, 17, 255, 4096, 65483, 65484, 65536, 65537, 200003, 1 << 20])
@pytest.mark.parametrize("F", [65536, 4096, 100])
def test_decode_memcpy_h2d_matches_oracle(size, F):
    cfg = ocfg(F=F)
    ctx = ctx_for(cfg)
    data = gen.random_bytes(size * 31 + F, size)
    w = O.encode_call(77, gen.PROC_H2D, [(O.K_U64, 0x1000), (O.K_OPAQUE_VAR, data.tobytes()), (O.K_U64, size)], cfg)
    ring = make_ring(1 << 21)
    head = (1 << 21) - 1000 - (size % 13)
    tail = place(ring, w, head)
    idx = ctx.index(1, 1 << 15, 64)
    idx.frame_scan([(ring, head, tail)])
    st = torch.zeros(1, dtype=torch.int32, device="cuda")
    cp = torch.zeros(1, dtype=torch.int64, device="cuda")
    for mis in (0, 1, 7, 12):
        buf, dst = dst_buffer(size, mis)
        idx.decode_memcpy_h2d(77, dst, size, st, cp)
        torch.cuda.synchronize()
        assert st.item() == O.OK and cp.item() == size
        host = buf.cpu().numpy()
        g0 = 64 + mis
        assert host[g0:g0 + size].tobytes() == data.tobytes()
        assert (host[:g0] == 0xA5).all() and (host[g0 + size:] == 0xA5).all()


def test_decode_memcpy_h2d_errors_match_oracle_and_leave_dst_untouched():
    cfg = ocfg(user={40: [O.K_U32]})
    ctx = ctx_for(cfg)
    good = gen.random_bytes(9, 5000).tobytes()
    cases = [
        O.frame(O.call_header(1, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0) + O.put_opaque_var(good) +
                O.put_u64(4999), 777),                                              # E_SIZE
        O.frame(O.call_header(2, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0) + O.put_opaque_var(good) +
                O.put_u64(5000) + b"\0\0\0\0", 900),                                # E_TRAILING
        O.frame(O.call_header(3, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0) + O.put_opaque_var(good[:5001 - 2]) +
                O.put_u64(4999), 900),                                              # ok (pad 1)
        O.frame(O.call_header(4, gen.PROG, 9, gen.PROC_H2D), 900),                  # E_RPC
        O.frame(O.call_header(5, gen.PROG, gen.VERS, 99), 900),                     # E_PROC
        O.frame(O.call_header(6, gen.PROG, gen.VERS, gen.PROC_H2D, (1, b"x" * 401)), 900),  # E_AUTH
        O.frame(O.call_header(7, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0) + O.put_u32(100), 900),  # TRUNC
        O.frame(O.call_header(8, gen.PROG, gen.VERS, 40) + O.put_u32(5), 900),      # E_PROC for h2d decode
        O.frame(b"\0\0\0", 900),                                                     # truncated xid
    ]
    bad_pad = bytearray(O.call_header(9, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0) + O.put_opaque_var(good[:3])
                        + O.put_u64(3))
    bad_pad[52 + 3] = 7
    cases.append(O.frame(bytes(bad_pad), 900))                                       # E_PAD
    ring = make_ring(1 << 16)
    tail = 0
    for w in cases:
        tail = place(ring, w, tail)
    idx = ctx.index(1, 1 << 10, 64)
    idx.frame_scan([(ring, 0, tail)])
    rb = ring_np(ring)
    s = O.frame_scan(rb, 0, tail)
    st = torch.zeros(1, dtype=torch.int32, device="cuda")
    cp = torch.zeros(1, dtype=torch.int64, device="cuda")
    for i, xid in enumerate([1, 2, 3, 4, 5, 6, 7, 8, 9]):
        L = O.record_logical(rb, s, i if xid != 9 else 9)
        c = O.parse_call(L, cfg)
        for cap in (6000, 10):
            want, data = O.decode_memcpy_h2d(L, c, cfg, cap)
            buf, dst = dst_buffer(6000, 0)
            idx.decode_memcpy_h2d(xid, dst, cap, st, cp)
            torch.cuda.synchronize()
            assert st.item() == want, (xid, cap, st.item(), want)
            host = buf.cpu().numpy()
            if want == O.OK:
                assert host[64:64 + len(data)].tobytes() == data and cp.item() == len(data)
            else:
                assert (host == 0xA5).all() and cp.item() == 0
    idx.decode_memcpy_h2d(0xDEAD, None, 0, st, cp)
    torch.cuda.synchronize()
    assert st.item() == O.E_XID
    lenient = ocfg(strict=False)
    lctx = ctx_for(lenient)
    lidx = lctx.index(1, 1 << 10, 64)
    lidx.frame_scan([(ring, 0, tail)])
    for xid, i in ((1, 0), (2, 1), (9, 9)):
        L = O.record_logical(rb, s, i)
        c = O.parse_call(L, lenient)
        want, data = O.decode_memcpy_h2d(L, c, lenient, 6000)
        buf, dst = dst_buffer(6000, 3)
        lidx.decode_memcpy_h2d(xid, dst, 6000, st, cp)
        torch.cuda.synchronize()
        assert st.item() == want and cp.item() == len(data)
        assert buf.cpu().numpy()[67:67 + len(data)].tobytes() == data


TYPES = [("i32", O.K_I32_VAR, np.int32), ("u32", O.K_U32_VAR, np.uint32), ("i64", O.K_I64_VAR, np.int64),
         ("u64", O.K_U64_VAR, np.uint64), ("f32", O.K_F32_VAR, np.float32), ("f64", O.K_F64_VAR, np.float64)]


@pytest.mark.parametrize("irregular", [False, True])
def test_decode_arrays_all_types_match_oracle(irregular):
    schema = [O.K_OPAQUE_VAR] + [k for _, k, _ in TYPES]
    cfg = ocfg(user={60: schema}, F=4096)
    ctx = ctx_for(cfg)
    g = gen.rng(60 + irregular)
    ring = make_ring(1 << 23)
    tail = 3
    recs = []
    for r in range(6):
        op = gen.random_bytes(r, int(g.integers(0, 3000)) | 1)
        arrays = [gen.random_elems(g, dt, int(g.integers(0, 40000))) for _, _, dt in TYPES]
        items = [(O.K_OPAQUE_VAR, op.tobytes())] + [(k, a) for (_, k, _), a in zip(TYPES, arrays)]
        L = O.call_header(600 + r, gen.PROG, gen.VERS, 60) + b"".join(O.encode_item(k, v) for k, v in items)
        w = O.frame_lens(L, gen.split_points(r + 17, len(L), 1, 9000)) if irregular else O.frame(L, 4096)
        tail = place(ring, w, tail)
        recs.append((op, arrays))
    idx = ctx.index(1, 1 << 14, 64)
    idx.frame_scan([(ring, 3, tail)])
    rb = ring_np(ring)
    s = compare_scan(idx.tables(), 0, rb, 3, tail, 1 << 14, 64)
    st = torch.zeros(1, dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    for r, (op, arrays) in enumerate(recs):
        L = O.record_logical(rb, s, r)
        c = O.parse_call(L, cfg)
        for a, (t, k, dt) in enumerate(TYPES):
            want_st, want = O.decode_item(L, c, a + 1, k, 1 << 20)
            out = torch.full((len(arrays[a]) + 2,), 0, dtype=crk.TYPED[t][1], device="cuda")
            idx.decode_array(t, 600 + r, a + 1, out, len(arrays[a]) + 2, cnt, st)
            torch.cuda.synchronize()
            assert st.item() == want_st == O.OK and cnt.item() == len(arrays[a])
            got = out.cpu().view(torch.uint8).numpy()[:len(want)]
            assert got.tobytes() == want.tobytes() == arrays[a].tobytes()
            # capacity one short -> E_SIZE, wrong type -> E_ARG
            if len(arrays[a]):
                idx.decode_array(t, 600 + r, a + 1, out, len(arrays[a]) - 1, cnt, st)
                torch.cuda.synchronize()
                assert st.item() == O.decode_item(L, c, a + 1, k, len(arrays[a]) - 1)[0] == O.E_SIZE
        wrong = "u32" if TYPES[0][0] != "u32" else "i32"
        out = torch.zeros(10, dtype=torch.int32, device="cuda")
        idx.decode_array("u32", 600 + r, 1, out, 1 << 20, cnt, st)
        torch.cuda.synchronize()
        assert st.item() == O.E_ARG
        ob = torch.zeros(len(op) + 5, dtype=torch.uint8, device="cuda")
        idx.decode_opaque(600 + r, 0, ob[1:], len(op), cnt, st)
        torch.cuda.synchronize()
        assert st.item() == O.OK and ob.cpu().numpy()[1:1 + len(op)].tobytes() == op.tobytes()


def test_decode_items_batch_c4_fixed_and_var():
    cfg = ocfg(user=gen.C4_SCHEMAS)
    ctx = ctx_for(cfg)
    calls = gen.c4_calls(3 << 20, max_count=1 << 14)
    ring = make_ring(1 << 23)
    tail = 0
    for c in calls:
        L = O.call_header(c.xid, gen.PROG, gen.VERS, c.proc) + b"".join(
            O.encode_item(k & 0xFF, v.tobytes() if (k & 0xFF) in (O.K_OPAQUE_VAR, O.K_OPAQUE_FIX) else v)
            for k, v in c.items)
        tail = place(ring, O.frame_lens(L, gen.split_points(gen.frag_seed(c), len(L))), tail)
    idx = ctx.index(1, 1 << 14, 1 << 10)
    idx.frame_scan([(ring, 0, tail)])
    rb = ring_np(ring)
    s = compare_scan(idx.tables(), 0, rb, 0, tail, 1 << 14, 1 << 10)
    compare_parse(idx.tables(), 0, rb, s, cfg)
    reqs, outs, expect = [], [], []
    status = torch.full((2000,), 99, dtype=torch.int32, device="cuda")
    counts = torch.zeros(2000, dtype=torch.int64, device="cuda")
    for i, c in enumerate(calls):
        L = O.record_logical(rb, s, i)
        oc = O.parse_call(L, cfg)
        for a, (code, v) in enumerate(c.items):
            k = code & 0xFF
            if k in (O.K_U32, O.K_U64):
                continue
            n = len(v)
            es = O.ELEM_SIZE[k]
            out = torch.zeros(n * es + 8, dtype=torch.uint8, device="cuda")
            j = len(reqs)
            reqs.append((c.xid, a, k, out.data_ptr(), n, counts.data_ptr() + 8 * j, status.data_ptr() + 4 * j))
            outs.append(out)
            expect.append(O.decode_item(L, oc, a, k, n))
    keep = idx.decode_items_batch(reqs)
    torch.cuda.synchronize()
    st = status.cpu().numpy()
    for j, (want_st, want) in enumerate(expect):
        assert st[j] == want_st == O.OK
        assert outs[j].cpu().numpy()[:len(want)].tobytes() == want.tobytes()
    del keep


def test_decode_memcpy_h2d_batch():
    cfg = ocfg()
    ctx = ctx_for(cfg)
    ring = make_ring(1 << 22)
    tail = 0
    datas = []
    for i in range(50):
        d = gen.random_bytes(i, int(gen.rng(i).integers(0, 40000)))
        datas.append(d)
        tail = place(ring, O.encode_call(i, gen.PROC_H2D, [(O.K_U64, 0), (O.K_OPAQUE_VAR, d.tobytes()),
                                                           (O.K_U64, len(d))], cfg, F=1500), tail)
    idx = ctx.index(1, 1 << 14, 256)
    idx.frame_scan([(ring, 0, tail)])
    bufs = [torch.zeros(len(d) + 32, dtype=torch.uint8, device="cuda") for d in datas]
    xids = torch.tensor(list(range(50)) + [999], dtype=torch.int32, device="cuda")
    dsts = torch.tensor([b.data_ptr() + (i % 16) for i, b in enumerate(bufs)] + [0], dtype=torch.int64, device="cuda")
    caps = torch.tensor([len(d) if i % 7 else len(d) - 1 for i, d in enumerate(datas)] + [0], dtype=torch.int64,
                        device="cuda")
    sts = torch.zeros(51, dtype=torch.int32, device="cuda")
    cps = torch.zeros(51, dtype=torch.int64, device="cuda")
    idx.decode_memcpy_h2d_batch(xids, dsts, caps, sts, cps)
    torch.cuda.synchronize()
    st = sts.cpu().numpy()
    for i, d in enumerate(datas):
        if i % 7 == 0 and len(d) > 0:
            assert st[i] == O.E_PTR
        else:
            assert st[i] == O.OK
            assert bufs[i].cpu().numpy()[i % 16:i % 16 + len(d)].tobytes() == d.tobytes()
    assert st[50] == O.E_XID


@pytest.mark.parametrize("host", [False, True])
def test_encode_call_matches_oracle(host):
    cfg = ocfg(F=3000)
    ctx = ctx_for(cfg)
    g = gen.rng(5)
    out = make_ring(1 << 20, host)
    cur = (1 << 20) - 12345
    for trial in range(25):
        items, oitems = [], []
        for _ in range(int(g.integers(0, 8))):
            k = int(g.choice([O.K_U32, O.K_U64, O.K_OPAQUE_VAR, O.K_I32_VAR, O.K_U64_VAR, O.K_F32_VAR, O.K_F64_VAR,
                              O.K_I64_VAR, O.K_U32_VAR, O.K_OPAQUE_FIX, O.K_F64_FIX]))
            if k == O.K_U32:
                v = int(g.integers(0, 1 << 32)); items.append((k, v)); oitems.append((k, v))
            elif k == O.K_U64:
                v = int(g.integers(0, 1 << 63)); items.append((k, v)); oitems.append((k, v))
            elif k in (O.K_OPAQUE_VAR, O.K_OPAQUE_FIX):
                d = gen.random_bytes(trial * 10 + len(items), int(g.integers(0, 9000)))
                items.append((k, torch.from_numpy(d).cuda())); oitems.append((k, d.tobytes()))
            else:
                dt = gen.NP_DTYPE[k]
                a = gen.random_elems(g, dt, int(g.integers(0, 3000)))
                t = torch.from_numpy(a.view(np.uint8).copy()).cuda().view(
                    {4: torch.int32, 8: torch.int64}[a.dtype.itemsize])
                items.append((k, t)); oitems.append((k, a))
        lens = None
        L = O.call_header(trial, gen.PROG, gen.VERS, 50) + b"".join(O.encode_item(k, v) for k, v in oitems)
        if trial % 3 == 1:
            lens = gen.split_points(trial, len(L), 0, 700) + [0]
            want = O.frame_lens(L, lens)
        else:
            want = O.frame(L, 3000)
        w = ctx.encode_call(trial, 50, items, out, cur, frag_lens=lens)
        assert w == len(want)
        torch.cuda.synchronize()
        assert out.read(cur, w) == want, trial
        cur += w + int(g.integers(0, 40))


@pytest.mark.parametrize("host", [False, True])
def test_encode_replies_match_oracle(host):
    cfg = ocfg(F=65536)
    ctx = ctx_for(cfg)
    out = make_ring(1 << 22, host)
    cur = (1 << 22) - 70001
    for n in (0, 1, 3, 4, 5, 15, 16, 17, 65503, 65504, 65505, 131041, 300007):
        d = gen.random_bytes(n, n)
        src = torch.zeros(n + 16, dtype=torch.uint8, device="cuda")
        for mis in (0, 5):
            src[mis:mis + n].copy_(torch.from_numpy(d))
            w = ctx.encode_memcpy_d2h(0x100 + n, src[mis:mis + n] if n else None, 0, out, cur, nbytes=n)
            want = O.encode_memcpy_d2h(0x100 + n, d.tobytes(), 0, 65536)
            torch.cuda.synchronize()
            assert w == len(want) and out.read(cur, w) == want, (n, mis)
            cur += w + 3
    w = ctx.encode_memcpy_d2h(7, None, 1, out, cur, nbytes=0)
    torch.cuda.synchronize()
    assert out.read(cur, w) == O.encode_memcpy_d2h(7, None, 1, 65536)
    cur += w
    g = gen.rng(3)
    for t, k, dt in TYPES:
        for n in (0, 1, 7, 4099, 40000):
            a = gen.random_elems(g, dt, n)
            src = torch.from_numpy(a.view(np.uint8).copy()).cuda().view(crk.TYPED[t][1]) if n else torch.empty(0, dtype=crk.TYPED[t][1], device="cuda")
            w = ctx.encode_array(t, 0x77, src, 0, out, cur)
            want = O.encode_array_reply(0x77, a, 0, 65536)
            torch.cuda.synchronize()
            assert out.read(cur, w) == want, (t, n)
            cur += w + 1


def test_encode_memcpy_d2h_batch_matches_oracle():
    cfg = ocfg(F=8192)
    ctx = ctx_for(cfg)
    out = make_ring(1 << 22)
    g = gen.rng(8)
    n = 40
    sizes = [int(g.integers(0, 30000)) for _ in range(n)]
    datas = [gen.random_bytes(i, s) for i, s in enumerate(sizes)]
    bufs = [torch.from_numpy(np.concatenate([np.zeros(i % 16, np.uint8), d])).cuda() for i, d in enumerate(datas)]
    srcs = torch.tensor([b.data_ptr() + i % 16 for i, b in enumerate(bufs)], dtype=torch.int64, device="cuda")
    errs = torch.tensor([1 if i % 9 == 4 else 0 for i in range(n)], dtype=torch.int32, device="cuda")
    xids = torch.arange(n, dtype=torch.int32, device="cuda") + 500
    nb = torch.tensor(sizes, dtype=torch.int64, device="cuda")
    offs = torch.zeros(n, dtype=torch.int64, device="cuda")
    tot = torch.zeros(1, dtype=torch.int64, device="cuda")
    start = (1 << 22) - 100000
    ctx.encode_memcpy_d2h_batch(xids, srcs, nb, errs, out, start, offs, tot)
    torch.cuda.synchronize()
    want = b"".join(O.encode_memcpy_d2h(500 + i, d.tobytes(), 1 if i % 9 == 4 else 0, 8192)
                    for i, d in enumerate(datas))
    assert tot.item() == len(want)
    assert out.read(start, len(want)) == want
    ow = np.cumsum([0] + [len(O.encode_memcpy_d2h(500 + i, d.tobytes(), 1 if i % 9 == 4 else 0, 8192))
                          for i, d in enumerate(datas)])[:-1]
    assert np.array_equal(offs.cpu().numpy(), ow + start)


_NP = {O.K_OPAQUE_VAR: np.uint8, O.K_OPAQUE_FIX: np.uint8, O.K_I32_VAR: np.int32, O.K_U32_VAR: np.uint32,
       O.K_F32_VAR: np.float32, O.K_I64_VAR: np.int64, O.K_U64_VAR: np.uint64, O.K_F64_VAR: np.float64,
       O.K_I32_FIX: np.int32, O.K_U32_FIX: np.uint32, O.K_F32_FIX: np.float32, O.K_I64_FIX: np.int64,
       O.K_U64_FIX: np.uint64, O.K_F64_FIX: np.float64}


@pytest.mark.parametrize("host,F", [(False, 4096), (True, 65536), (False, 1 << 20)])
def test_encode_replies_batch_matches_oracle(host, F):
    """Generic batched REPLY encoder (NEXT-3) vs or_encode_reply_item, every kind, err != 0, unknown kind,
    misaligned sources, multi-fragment records and ring wrap."""
    ctx = ctx_for(ocfg(F=F))
    out = crk.Ring.host(1 << 21) if host else make_ring(1 << 21)
    g = gen.rng(31)
    reqs, want, keep = [], [], []
    for i in range(90):
        kind = [0, O.K_U32, O.K_U64, 99, *range(3, 17)][i % 18]
        err = 3 if i % 13 == 5 else 0
        xid = 9000 + i
        value = int(g.integers(0, 1 << 63)) * 2 + (i & 1)
        src, count, elems = None, 0, None
        if kind in _NP:
            count = int(g.integers(0, [1, 7, 300, 20000][i % 4]))
            elems = gen.random_elems(g, _NP[kind], count)
            es = np.dtype(_NP[kind]).itemsize
            mis = (i * 4) % 16 if es > 1 else i % 16  # misaligned 8-byte sources -> err = E_ARG
            raw = np.concatenate([np.zeros(mis, np.uint8), elems.view(np.uint8)])
            t = torch.from_numpy(raw).cuda()
            keep.append(t)
            src = t.data_ptr() + mis
        reqs.append((xid, err, kind, value, src, count))
        eff = O.E_ARG if err == 0 and elems is not None and mis % es else err
        want.append(O.encode_reply_item(xid, eff, kind if kind != 99 else 0, value, elems, F))
    reqs.append((9999, 0, O.K_U32_VAR, 0, None, 5))  # count > 0 with no source -> err = E_ARG
    want.append(O.encode_reply_item(9999, O.E_ARG, O.K_U32_VAR, 0, None, F))
    offs = torch.zeros(len(reqs), dtype=torch.int64, device="cuda")
    tot = torch.zeros(1, dtype=torch.int64, device="cuda")
    start = (1 << 21) - 70000
    ctx.encode_replies_batch(reqs, out, start, offs, tot)
    torch.cuda.synchronize()
    allw = b"".join(want)
    assert tot.item() == len(allw)
    got = out.read(start, len(allw))
    pos = 0
    for i, w in enumerate(want):
        assert got[pos:pos + len(w)] == w, f"reply {i} kind {reqs[i][2]} err {reqs[i][1]} count {reqs[i][5]}"
        pos += len(w)
    assert np.array_equal(offs.cpu().numpy(), np.cumsum([0] + [len(w) for w in want])[:-1] + start)


MOVER_CONFIGS = [{}, {"mover_tail_tiles": 0, "mover_reserve_ctas": 16},
                 {"mover_tail_tiles": 64, "mover_run": 1, "tile_bytes": 4096}, {"mover_tail_tiles": 1, "mover_run": 64},
                 # small tiles and short runs: the batch holds >= 2 runs per CTA, so run_map_kernel's run -> job
                 # map drives the claims (with and without the single-tile tail region)
                 {"tile_bytes": 4096, "mover_run": 2, "mover_tail_tiles": 0},
                 {"tile_bytes": 4096, "mover_run": 2, "mover_tail_tiles": 1, "mover_reserve_ctas": 16},
                 # the fused single-CTA front end (scan + parse + plan in one launch) on the same batch
                 {"fused_front_max_records": 1024, "fused_front_max_window": 1 << 40}]


@pytest.mark.parametrize("host,mover", [(False, m) for m in range(len(MOVER_CONFIGS))] + [(True, 0), (True, 6)])
def test_serve_matches_oracle(host, mover):
    cfg = ocfg(F=16384)
    ctx = ctx_for(cfg, **MOVER_CONFIGS[mover])
    streams, region_bytes = gen.c5_endpoint(0, n_streams=4, payload_per_stream=3 << 20, h2d_budget=2 << 20,
                                            lo=1, hi=1 << 20, misalign=True)
    region = torch.zeros(region_bytes + 64, dtype=torch.uint8, device="cuda")
    base = region.data_ptr()
    rings, sends, offs = [], [], []
    host_region = np.zeros(region_bytes + 64, np.uint8)
    for s in streams:
        ring = make_ring(1 << 22, host)
        cur = 100 * s.stream
        for r in s.records:
            if r.kind == gen.PROC_D2H:
                d = gen.random_bytes(r.seed & 0xFFFFFFFF, r.size)
                host_region[r.region_off:r.region_off + r.size] = d
        for i, r in enumerate(s.records):
            if r.kind == gen.PROC_H2D:
                d = gen.random_bytes(r.seed & 0xFFFFFFFF, r.size)
                c = h2d_call(r.xid, d, base + r.region_off)
            else:
                c = d2h_call(r.xid, base + r.region_off, r.size)
            cur = place(ring, O.encode_call(*c, cfg, F=16384), cur)
        # error records: a duplicate xid, an out-of-region pointer, a malformed record
        dup = s.records[0]
        cur = place(ring, O.encode_call(*h2d_call(dup.xid, np.zeros(8, np.uint8), base), cfg), cur)
        cur = place(ring, O.encode_call(*d2h_call(0xE0000000 + s.stream, base + region_bytes + 64, 16), cfg), cur)
        cur = place(ring, O.encode_call(*h2d_call(0xE1000000 + s.stream, np.ones(8, np.uint8), base - 8), cfg), cur)
        cur = place(ring, O.frame(O.call_header(0xE2000000, gen.PROG, 3, 1), 100), cur)
        rings.append((ring, 100 * s.stream, cur))
        sends.append(make_ring(1 << 23, host))
        offs.append(777 * s.stream)
    region.copy_(torch.from_numpy(host_region))
    # the run -> job map configs need the multi-kernel planning path: an index above kSmallServe (1024)
    # records, otherwise the one-block planner plans the jobs and the mover claims through find_job
    map_cfg = MOVER_CONFIGS[mover].get("mover_run") == 2
    max_records = 1 << 11 if map_cfg else 1 << 10
    idx = ctx.index(4, 1 << 14, max_records)
    idx.serve(rings, sends, offs, base, region_bytes + 64)
    torch.cuda.synchronize()
    if map_cfg:
        assert ctx.debug_counters()[13] == 1, "the mover did not claim through the run -> job map"
    T = idx.tables(4)
    ring_bytes = [ring_np(r[0]) for r in rings]
    want = O.serve([(rb, h, t) for rb, (_, h, t) in zip(ring_bytes, rings)], cfg, host_region, base,
                   [1 << 23] * 4, offs, max_frags_per_ring=(1 << 14) // 4, max_records_per_ring=max_records // 4)
    assert np.array_equal(region.cpu().numpy(), host_region)
    P = T["parsed"]
    assert [r["status"] for r in want["records"]] == list(P["serve_status"])
    assert [r["reply_err"] for r in want["records"]] == list(P["serve_reply_err"])
    assert [r["reply_off"] for r in want["records"] if r["reply_err"] >= 0] == \
           [int(o) for o, e in zip(P["serve_reply_off"], P["serve_reply_err"]) if e >= 0]
    for r in range(4):
        assert T["rings"][r]["reply_bytes"] == want["reply_bytes"][r]
        assert T["rings"][r]["consumed"] == want["consumed"][r]
        n = want["reply_bytes"][r]
        assert sends[r].read(offs[r], n) == bytes(want["send"][r][offs[r]:offs[r] + n])


def test_ring_copy_and_async_results():
    g = gen.rng(21)
    for (cd, cs) in [(1 << 12, 1 << 12), (1 << 12, 1 << 14), (1 << 14, 1 << 12)]:
        src = crk.Ring.host(cs)
        src.host_view()[:] = gen.random_bytes(cs, cs)
        dst = crk.Ring.device(cd)
        dst.tensor().fill_(0)
        for _ in range(5):
            head = int(g.integers(0, 1 << 20))
            n = int(g.integers(0, min(cd, cs) + 1))
            crk.ring_copy(dst, src, head, head + n)
            torch.cuda.synchronize()
            assert dst.read(head, n) == src.read(head, n)
            back = crk.Ring.host(cs)
            crk.ring_copy(back, dst, head, head + n)
            torch.cuda.synchronize()
            assert back.read(head, n) == src.read(head, n)
    with pytest.raises(crk.CrkError):
        crk.ring_copy(dst, src, 0, max(cd, cs) + 1)
    cfg = ocfg()
    ctx = ctx_for(cfg)
    ring = make_ring(1 << 16)
    w = O.encode_call(1, gen.PROC_H2D, [(O.K_U64, 0), (O.K_OPAQUE_VAR, b"abc"), (O.K_U64, 3)], cfg)
    ring.write(0, w)
    idx = ctx.index(2, 1024, 64)
    idx.frame_scan([(ring, 0, len(w)), (ring, 0, 3)])
    out = crk.PinnedResults(2)
    idx.ring_results_async(out)
    torch.cuda.synchronize()
    rows = out.rows()
    assert rows == idx.ring_results(2)
    assert rows[0]["status"] == O.OK and rows[0]["n_records"] == 1 and rows[1]["status"] == O.INCOMPLETE


@pytest.mark.parametrize("strict,fused", [(True, False), (False, False), (True, True), (False, True)])
def test_serve_cred_bodies_lenient_and_duplicates_match_oracle(strict, fused):
    """Non-empty cred/verf bodies (args start past the prefetched head), odd pads, lenient mode; through the
    separate scan / parse / plan kernels and through the fused single-CTA front end."""
    cfg = ocfg(strict=strict, F=3000)
    ctx = ctx_for(cfg, fused_front_max_records=1024 if fused else 0)
    region = torch.zeros(1 << 20, dtype=torch.uint8, device="cuda")
    base = region.data_ptr()
    host_region = np.zeros(1 << 20, np.uint8)
    host_region[500000:600000] = gen.random_bytes(4, 100000)
    region.copy_(torch.from_numpy(host_region))
    g = gen.rng(31)
    wires = []
    for i in range(40):
        cl, vl = int(g.integers(0, 401)), int(g.integers(0, 401))
        cred = (1, gen.random_bytes(i, cl).tobytes())
        verf = (6, gen.random_bytes(i + 99, vl).tobytes())
        if i % 3 == 0:
            L = O.call_header(100 + i, gen.PROG, gen.VERS, gen.PROC_D2H, cred, verf) + O.put_u64(base + 500000 + i) + \
                O.put_u64(int(g.integers(0, 90000)))
        else:
            n = int(g.integers(0, 5000))
            size = n if i % 5 else n + 3          # strict: E_SIZE; lenient: copies min(n, size)
            L = O.call_header(100 + i, gen.PROG, gen.VERS, gen.PROC_H2D, cred, verf) + O.put_u64(base + 7000 * i) + \
                O.put_opaque_var(gen.random_bytes(i + 7, n).tobytes()) + O.put_u64(size)
            if i % 7 == 0:
                L += b"\0" * 8                     # trailing bytes: strict E_TRAILING, lenient ignored
        wires.append(O.frame(L, int(g.integers(7, 3000))))
    wires.append(wires[5])                         # duplicate xid (reading R11)
    ring = make_ring(1 << 21)
    tail = 0
    for w in wires:
        tail = place(ring, w, tail)
    send = make_ring(1 << 22)
    idx = ctx.index(1, 1 << 14, 256)
    idx.serve([(ring, 0, tail)], [send], [40], base, region.numel())
    torch.cuda.synchronize()
    T = idx.tables(1)
    want = O.serve([(ring_np(ring), 0, tail)], cfg, host_region, base, [1 << 22], [40], max_frags_per_ring=1 << 14,
                   max_records_per_ring=256)
    assert [r["status"] for r in want["records"]] == list(T["parsed"]["serve_status"])
    assert [r["reply_err"] for r in want["records"]] == list(T["parsed"]["serve_reply_err"])
    assert np.array_equal(region.cpu().numpy(), host_region)
    n = want["reply_bytes"][0]
    assert T["rings"][0]["reply_bytes"] == n
    assert send.read(40, n) == bytes(want["send"][0][40:40 + n])


def test_ctx_rejects_bad_mover_config():
    for kw in ({"mover_tail_tiles": 65}, {"mover_reserve_ctas": 10 ** 6}, {"mover_run": 0}):
        with pytest.raises(crk.CrkError) as e:
            crk.Context(0, **kw)
        assert e.value.status == crk.E_ARG


def test_serve_rejects_index_larger_than_job_scratch():
    ctx = crk.Context(0, max_jobs=64)
    idx = ctx.index(1, 256, 64)  # serve needs 2 jobs per record
    ring = make_ring(1 << 12)
    with pytest.raises(crk.CrkError) as e:
        idx.serve([(ring, 0, 0)], [make_ring(1 << 12)], [0], 0, 0)
    assert e.value.status == crk.E_CAPACITY


def test_staged_e2e_path_matches_oracle():
    """Copy-engine mode: host ring -> crk_ring_copy -> serve from HBM -> crk_ring_copy replies -> host."""
    cfg = ocfg(F=8192)
    ctx = ctx_for(cfg)
    region = torch.zeros(1 << 22, dtype=torch.uint8, device="cuda")
    base = region.data_ptr()
    host_region = np.zeros(1 << 22, np.uint8)
    host_region[1 << 21:(1 << 21) + 300000] = gen.random_bytes(8, 300000)
    region.copy_(torch.from_numpy(host_region))
    hring, dring = crk.Ring.host(1 << 20), crk.Ring.device(1 << 20)
    head = (1 << 20) - 5000
    cur = head
    for i in range(12):
        if i % 2:
            c = d2h_call(i + 1, base + (1 << 21) + 1000 * i, 20000 + 977 * i)
        else:
            c = h2d_call(i + 1, gen.random_bytes(i, 30000 + 311 * i), base + 40000 * i)
        cur = place(hring, O.encode_call(*c, cfg, F=8192), cur)
    hsend, dsend = crk.Ring.host(1 << 20), crk.Ring.device(1 << 20)
    crk.ring_copy(dring, hring, head, cur)
    idx = ctx.index(1, 1024, 64)
    idx.serve([(dring, head, cur)], [dsend], [77], base, region.numel())
    res = crk.PinnedResults(1)
    idx.ring_results_async(res)
    torch.cuda.synchronize()
    n = res.rows()[0]["reply_bytes"]
    crk.ring_copy(hsend, dsend, 77, 77 + n)
    torch.cuda.synchronize()
    want = O.serve([(hring.host_view().copy(), head, cur)], cfg, host_region, base, [1 << 20], [77])
    assert n == want["reply_bytes"][0]
    assert hsend.read(77, n) == bytes(want["send"][0][77:77 + n])
    assert np.array_equal(region.cpu().numpy(), host_region)


@pytest.mark.parametrize("shape,out0", [((4096, 256), 5), ((64, 16), 8)])
def test_serve_graph_replays_with_doorbell_cursors(shape, out0):
    """A captured serve step replayed over successive windows of the same ring == the oracle per window.  The
    small index with an aligned send cursor takes the fused front end's lean path, its cursors read from the
    doorbell at replay time (the mover then finds an empty plan)."""
    cfg = ocfg(F=4096)
    ctx = ctx_for(cfg, lean_backoff=0)
    region = torch.zeros(1 << 20, dtype=torch.uint8, device="cuda")
    base = region.data_ptr()
    host_region = np.zeros(1 << 20, np.uint8)
    host_region[600000:700000] = gen.random_bytes(2, 100000)
    region.copy_(torch.from_numpy(host_region))
    ring = make_ring(1 << 16)
    send = make_ring(1 << 17)
    idx = ctx.index(1, *shape)
    bell = crk.HostBuffer(3 * 8)
    cells = bell.np.view(np.uint64)
    graph = idx.serve_graph([ring], [send], base, region.numel(), bell)
    head, out = 60000, out0
    for batch in range(4):
        wires = []
        for i in range(3):
            xid = 1000 * batch + i
            if i == 1:
                wires.append(O.encode_call(*d2h_call(xid, base + 600000 + 999 * batch, 3000 + 1000 * batch), cfg,
                                           F=4096))
            else:
                wires.append(O.encode_call(*h2d_call(xid, gen.random_bytes(xid, 2000 + 777 * i),
                                                     base + 10000 * (batch * 3 + i)), cfg, F=4096))
        w = b"".join(wires)
        tail = place(ring, w, head)
        cells[:] = [head, tail, out]
        torch.cuda.synchronize()
        graph.launch()
        torch.cuda.synchronize()
        res = idx.ring_results(1)[0]
        want = O.serve([(ring_np(ring), head, tail)], cfg, host_region, base, [1 << 17], [out])
        assert res["status"] == O.OK and res["consumed"] == tail and res["reply_bytes"] == want["reply_bytes"][0]
        n = want["reply_bytes"][0]
        assert send.read(out, n) == bytes(want["send"][0][out:out + n])
        assert np.array_equal(region.cpu().numpy(), host_region)
        if out0 % 4 == 0:
            assert ctx.debug_counters()[1] == 0  # the lean path served it
        head, out = tail, out + n
    cells[:] = [10, 5, 0]  # invalid window: E_ARG, nothing served
    graph.launch()
    torch.cuda.synchronize()
    assert idx.ring_results(1)[0]["status"] == O.E_ARG
    graph.close()


def test_batch_requests_reject_null_and_misaligned_dst():
    """batched requests check their destinations like the single-request calls do (include/crk.h:
    NULL dst with a non-empty payload, or a typed dst not aligned to the element size -> E_ARG, nothing
    written) instead of faulting or byte-swapping across element lanes."""
    cfg = ocfg(user={33: [O.K_I32_VAR, O.K_F64_VAR, O.K_OPAQUE_VAR]})
    ctx = ctx_for(cfg)
    ring = make_ring(1 << 16)
    a = np.arange(9, dtype=np.int32)
    b = np.arange(3, dtype=np.float64)
    wire = (O.encode_call(1, 33, [(O.K_I32_VAR, a), (O.K_F64_VAR, b), (O.K_OPAQUE_VAR, b"")], cfg)
            + O.encode_call(2, gen.PROC_H2D, [(O.K_U64, 0), (O.K_OPAQUE_VAR, b"abcdef"), (O.K_U64, 6)], cfg))
    tail = place(ring, wire, 0)
    idx = ctx.index(1, 64, 16)
    idx.frame_scan([(ring, 0, tail)])
    out = torch.zeros(256, dtype=torch.uint8, device="cuda")
    st = torch.full((6,), 99, dtype=torch.int32, device="cuda")
    p = out.data_ptr()
    reqs = [(1, 0, O.K_I32_VAR, p + 2, 9, None, st.data_ptr()),        # misaligned int32 dst
            (1, 1, O.K_F64_VAR, p + 4, 3, None, st.data_ptr() + 4),    # misaligned double dst
            (1, 0, O.K_I32_VAR, 0, 9, None, st.data_ptr() + 8),        # NULL dst, 9 elements
            (1, 2, O.K_OPAQUE_VAR, 0, 0, None, st.data_ptr() + 12),    # NULL dst, empty opaque: fine
            (1, 1, O.K_F64_VAR, p + 64, 3, None, st.data_ptr() + 16)]  # aligned: decoded
    keep = idx.decode_items_batch(reqs)
    torch.cuda.synchronize()
    assert st.cpu().tolist()[:5] == [O.E_ARG, O.E_ARG, O.E_ARG, O.OK, O.OK]
    got = out.cpu().numpy()
    assert not got[:64].any()  # nothing written by the rejected requests
    assert got[64:88].tobytes() == b.tobytes()
    del keep
    xids = torch.tensor([2, 2], dtype=torch.int32, device="cuda")
    dsts = torch.tensor([0, p + 100], dtype=torch.int64, device="cuda")
    caps = torch.tensor([6, 6], dtype=torch.int64, device="cuda")
    sts = torch.full((2,), 99, dtype=torch.int32, device="cuda")
    cps = torch.full((2,), 99, dtype=torch.int64, device="cuda")
    idx.decode_memcpy_h2d_batch(xids, dsts, caps, sts, cps)
    torch.cuda.synchronize()
    assert sts.cpu().tolist() == [O.E_ARG, O.OK] and cps.cpu().tolist() == [0, 6]
    assert out.cpu().numpy()[100:106].tobytes() == b"abcdef"
