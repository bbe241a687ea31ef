"""Pins the oracle to things other than itself (CPU only).

* RFC 4506 §7 worked example (tests/golden/rfc4506_sec7_file.hex).
* Python's xdrlib (an independent XDR implementation) for every primitive encode and typed decode.
* numpy big-endian dtype views for typed-array decode (RFC 4506 §4.1-4.7, §4.12-4.13).
* Brute force: every fragment split of tiny records, with zero-length fragments inserted (RFC 5531 §11).
* Closed forms: wire sizes and the physical offset of payload bytes.
* Every status code, each from a crafted stream.
* Round trips and invariants (hypothesis).
"""
import itertools
import struct
import warnings

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import gen

with warnings.catch_warnings():
    warnings.simplefilter("ignore", DeprecationWarning)
    import xdrlib

CFG = O.Config(prog=gen.PROG, vers=gen.VERS, proc_h2d=gen.PROC_H2D, proc_d2h=gen.PROC_D2H)


def ring_of(wire: bytes, cap: int | None = None, at: int = 0) -> np.ndarray:
    cap = cap or 1 << max(6, (len(wire) + at).bit_length())
    r = np.zeros(cap, np.uint8)
    for i, b in enumerate(wire):
        r[(at + i) % cap] = b
    return r


def hdr(n, last):
    return struct.pack(">I", n | (0x80000000 if last else 0))


# ------------------------------------------------------------------ RFC 4506 §7

def test_rfc4506_sec7_example(golden_dir):
    words = [ln.strip() for ln in open(f"{golden_dir}/rfc4506_sec7_file.hex") if ln.strip() and ln[0] != "#"]
    gold = bytes.fromhex("".join(words))
    assert len(gold) == 48
    enc = (O.put_opaque_var(b"sillyprog") + O.put_u32(2) + O.put_opaque_var(b"lisp") + O.put_opaque_var(b"john")
           + O.put_opaque_var(b"(quit)"))
    assert enc == gold
    p = xdrlib.Packer()
    p.pack_string(b"sillyprog"); p.pack_enum(2); p.pack_string(b"lisp"); p.pack_string(b"john")
    p.pack_opaque(b"(quit)")
    assert p.get_buffer() == gold


# ------------------------------------------------------------------ xdrlib cross-checks

@given(st.integers(0, 2**32 - 1))
def test_u32_vs_xdrlib(v):
    p = xdrlib.Packer(); p.pack_uint(v)
    assert O.put_u32(v) == p.get_buffer()


@given(st.integers(0, 2**64 - 1))
def test_u64_vs_xdrlib(v):
    p = xdrlib.Packer(); p.pack_uhyper(v)
    assert O.put_u64(v) == p.get_buffer()


@given(st.binary(max_size=70))
def test_opaque_vs_xdrlib(b):
    p = xdrlib.Packer(); p.pack_opaque(b)
    assert O.put_opaque_var(b) == p.get_buffer()
    q = xdrlib.Packer(); q.pack_fopaque(len(b), b)
    assert O.put_opaque_fix(b) == q.get_buffer()


@pytest.mark.parametrize("dtype,pack", [(np.int32, "pack_int"), (np.uint32, "pack_uint"), (np.int64, "pack_hyper"),
                                        (np.uint64, "pack_uhyper"), (np.float32, None), (np.float64, None)])
def test_arrays_vs_xdrlib(dtype, pack):
    g = gen.rng(99)
    a = gen.random_elems(g, dtype, 257)
    p = xdrlib.Packer()
    if pack is None:  # floats: pack the bit pattern through the same-width unsigned packer (reading R13)
        u = a.view(np.uint32 if dtype == np.float32 else np.uint64)
        fn = p.pack_uint if dtype == np.float32 else p.pack_uhyper
        p.pack_array([int(x) for x in u], fn)
    else:
        p.pack_array([int(x) for x in a], getattr(p, pack))
    assert O.put_array(a, with_count=True) == p.get_buffer()
    q = xdrlib.Packer()
    if pack is None:
        u = a.view(np.uint32 if dtype == np.float32 else np.uint64)
        q.pack_farray(len(u), [int(x) for x in u], q.pack_uint if dtype == np.float32 else q.pack_uhyper)
    else:
        q.pack_farray(len(a), [int(x) for x in a], getattr(q, pack))
    assert O.put_array(a, with_count=False) == q.get_buffer()


def test_float_values_vs_xdrlib():
    # ordinary values through xdrlib's own float path (struct '>f' / '>d')
    vals = [0.0, -0.0, 1.0, -2.5, 3.2, 1e-30, 6.02e23]
    p = xdrlib.Packer(); p.pack_array(vals, p.pack_double)
    assert O.put_array(np.array(vals, np.float64)) == p.get_buffer()
    p = xdrlib.Packer(); p.pack_array(vals, p.pack_float)
    assert O.put_array(np.array(vals, np.float32)) == p.get_buffer()


# ------------------------------------------------------------------ typed decode vs numpy / xdrlib

@pytest.mark.parametrize("kind", [O.K_I32_VAR, O.K_U32_VAR, O.K_F32_VAR, O.K_I64_VAR, O.K_U64_VAR, O.K_F64_VAR])
def test_typed_decode_vs_numpy_and_xdrlib(kind):
    dt = gen.NP_DTYPE[kind]
    es = np.dtype(dt).itemsize
    a = gen.random_elems(gen.rng(kind), dt, 1000)
    # the CALL is assembled with xdrlib (independent encoder)
    p = xdrlib.Packer()
    p.pack_uint(0x55); p.pack_uint(0); p.pack_uint(2); p.pack_uint(CFG.prog); p.pack_uint(CFG.vers); p.pack_uint(33)
    p.pack_uint(0); p.pack_opaque(b""); p.pack_uint(0); p.pack_opaque(b"")
    u = a.view(np.uint32 if es == 4 else np.uint64)
    p.pack_array([int(x) for x in u], p.pack_uint if es == 4 else p.pack_uhyper)
    L = p.get_buffer()
    cfg = O.Config(prog=CFG.prog, vers=CFG.vers, user_schemas={33: [kind]})
    c = O.parse_call(L, cfg)
    assert c.status == O.OK and c.count[0] == 1000 and c.off[0] == 44
    stt, out = O.decode_item(L, c, 0, kind, 1000)
    assert stt == O.OK
    be = np.frombuffer(L[44:], dtype=">u4" if es == 4 else ">u8")
    assert np.array_equal(out.view(np.uint32 if es == 4 else np.uint64), be.astype(be.dtype.newbyteorder("=")))
    assert out.tobytes() == a.tobytes()  # bit-exact incl. NaN payloads, -0, denormals (reading R13)
    up = xdrlib.Unpacker(L[40:])
    vals = up.unpack_array(up.unpack_uint if es == 4 else up.unpack_uhyper)
    assert [int(x) for x in out.view(np.uint32 if es == 4 else np.uint64)] == vals


# ------------------------------------------------------------------ brute force over fragment splits

def compositions(n):
    for mask in range(1 << max(0, n - 1)):
        cuts = [i + 1 for i in range(n - 1) if mask >> i & 1]
        yield [b - a for a, b in zip([0] + cuts, cuts + [n])]


@pytest.mark.parametrize("n", list(range(0, 11)))
def test_every_split_with_zero_fragments(n):
    """Every composition of an n-byte record into fragments, plus up to two zero-length fragments at any
    position (RFC 5531 §11; reading R1/R2), decodes to the same logical bytes and prefix sums."""
    L = bytes((i * 37 + 11) & 0xFF for i in range(n))
    base = list(compositions(n)) if n else [[0]]
    count = 0
    for lens in base:
        variants = [lens]
        if len(lens) <= 4:
            for pos in range(len(lens) + 1):
                variants.append(lens[:pos] + [0] + lens[pos:])
            for p1, p2 in itertools.combinations(range(len(lens) + 2), 2):
                v = list(lens)
                v.insert(p1, 0)
                v.insert(p2, 0)
                variants.append(v)
        for v in variants:
            wire = b"".join(hdr(ln, i == len(v) - 1) + L[sum(v[:i]):sum(v[:i + 1])] for i, ln in enumerate(v))
            for at in (0, 61):  # also across the ring wrap (reading R16)
                ring = ring_of(wire, 64, at)
                s = O.frame_scan(ring, at, at + len(wire))
                assert s.status == O.OK and s.consumed == at + len(wire)
                assert len(s.recs) == 1 and s.recs[0]["len"] == n and s.recs[0]["nfrags"] == len(v)
                assert [f["len"] for f in s.frags] == v
                assert [f["lstart"] for f in s.frags] == list(np.cumsum([0] + v[:-1]))
                assert [f["last"] for f in s.frags] == [0] * (len(v) - 1) + [1]
                assert O.record_logical(ring, s, 0) == L
                count += 1
    assert count > 0


def test_splits_of_a_real_call_three_fragments():
    """All cut pairs of a real ~72-byte memcpy CALL into <= 3 fragments parse identically."""
    data = bytes(range(17))
    w = O.encode_call(0xABC, gen.PROC_H2D, [(O.K_U64, 0x1000), (O.K_OPAQUE_VAR, data), (O.K_U64, 17)], CFG,
                      F=1 << 20)
    L = w[4:]
    n = len(L)
    ref = O.parse_call(L, CFG)
    assert ref.status == O.OK
    for a in range(0, n + 1, 3):
        for b in range(a, n + 1, 5):
            lens = [x for x in (a, b - a, n - b)]
            wire = b"".join(hdr(ln, i == 2) + L[sum(lens[:i]):sum(lens[:i + 1])] for i, ln in enumerate(lens))
            ring = ring_of(wire, 256)
            s = O.frame_scan(ring, 0, len(wire))
            Lr = O.record_logical(ring, s, 0)
            assert Lr == L
            c = O.parse_call(Lr, CFG)
            st_, out = O.decode_memcpy_h2d(Lr, c, CFG, 64)
            assert st_ == O.OK and out == data


# ------------------------------------------------------------------ closed forms

def test_closed_form_wire_sizes():
    F = 65536
    # C3 1 GiB HtoD record: logical 2^30 + 60 -> 16,385 fragments, 1,073,807,424 wire bytes
    assert O.frame_count((1 << 30) + 60, F) == 16385
    assert O.wire_size((1 << 30) + 60, F) == 1_073_807_424
    # C3 1 GiB DtoH reply: logical 2^30 + 32
    assert O.wire_size((1 << 30) + 32, F) == 1_073_807_396
    # C2: A 409,600 / B 819,200 HtoD, C 819,200 DtoH
    assert O.wire_size(409_600 + 60, F) == 409_688
    assert O.wire_size(819_200 + 60, F) == 819_312
    assert O.wire_size(819_200 + 32, F) == 819_284
    # C1 logical 8,256 B -> one fragment, 8,260 wire bytes
    c1 = gen.c1_call()
    cfg = O.Config(prog=gen.PROG, vers=gen.VERS, user_schemas={gen.PROC_C1: gen.C1_SCHEMA})
    w = O.encode_call(c1.xid, c1.proc, c1.items, cfg)
    assert len(w) == 8260
    for n in (0, 1, 4, 65535, 65536, 65537, 131072):  # reading R3: no empty trailing fragment
        assert O.frame_count(n, F) == max(1, -(-n // F))


def test_closed_form_payload_physical_offsets():
    """phys(i) = r0 + 52 + i + 4 * (floor((52 + i) / F) + 1) for a greedily framed HtoD CALL."""
    F = 4096
    n = 3 * F + 123
    data = gen.random_bytes(5, n)
    w = O.encode_call(1, gen.PROC_H2D, [(O.K_U64, 0), (O.K_OPAQUE_VAR, data), (O.K_U64, n)], CFG, F=F)
    r0 = 1000
    ring = ring_of(w, 1 << 15, r0)
    s = O.frame_scan(ring, r0, r0 + len(w))
    assert s.status == O.OK
    for i in (0, F - 53, F - 52, 2 * F, n - 1):
        phys = r0 + 52 + i + 4 * ((52 + i) // F + 1)
        assert ring[phys % len(ring)] == data[i]
        f = next(f for f in s.frags if f["lstart"] <= 52 + i < f["lstart"] + f["len"])
        assert f["phys"] + (52 + i - f["lstart"]) == phys


# ------------------------------------------------------------------ status codes

def call_logical(xid=7, proc=gen.PROC_H2D, data=b"abcde", size=None, cred=(0, b""), extra=b"", mtype=0,
                 rpcvers=2, prog=None, vers=None):
    p = xdrlib.Packer()
    p.pack_uint(xid); p.pack_uint(mtype); p.pack_uint(rpcvers); p.pack_uint(CFG.prog if prog is None else prog)
    p.pack_uint(CFG.vers if vers is None else vers); p.pack_uint(proc)
    p.pack_uint(cred[0]); p.pack_opaque(cred[1]); p.pack_uint(0); p.pack_opaque(b"")
    p.pack_uhyper(0x1000); p.pack_opaque(data); p.pack_uhyper(len(data) if size is None else size)
    return p.get_buffer() + extra


def status_of(L, cfg=CFG, dst=1 << 20):
    c = O.parse_call(L, cfg)
    return O.decode_memcpy_h2d(L, c, cfg, dst)[0]


def test_status_codes_parse():
    assert status_of(call_logical()) == O.OK
    assert status_of(call_logical()[:3]) == O.E_TRUNCATED
    assert status_of(call_logical()[:50]) == O.E_TRUNCATED
    assert status_of(call_logical(mtype=1)) == O.E_RPC
    assert status_of(call_logical(rpcvers=3)) == O.E_RPC
    assert status_of(call_logical(prog=5)) == O.E_RPC
    assert status_of(call_logical(vers=9)) == O.E_RPC
    assert status_of(call_logical(proc=99)) == O.E_PROC
    assert status_of(call_logical(cred=(1, b"x" * 400))) == O.OK
    assert status_of(call_logical(cred=(1, b"x" * 401))) == O.E_AUTH
    assert status_of(call_logical(size=4)) == O.E_SIZE
    assert status_of(call_logical(extra=b"\0\0\0\0")) == O.E_TRAILING
    assert status_of(call_logical(), dst=4) == O.E_PTR
    assert status_of(call_logical(data=b""), dst=0) == O.OK  # reading R14: opaque n = 0
    # nonzero pad byte after a 5-byte opaque (data at 52..57, pad 57..60)
    L = bytearray(call_logical()); L[58] = 1
    assert status_of(bytes(L)) == O.E_PAD
    lenient = O.Config(prog=CFG.prog, vers=CFG.vers, strict=False)
    assert status_of(bytes(L), lenient) == O.OK  # reading R5
    assert status_of(call_logical(extra=b"\0\0\0\0"), lenient) == O.OK
    # lenient E_SIZE reading (R9): copies min(n, size)
    L2 = call_logical(size=3)
    c = O.parse_call(L2, lenient)
    assert O.decode_memcpy_h2d(L2, c, lenient, 100) == (O.OK, b"abc")
    # first failure in logical order wins: bad rpcvers beats a later bad pad
    L3 = bytearray(call_logical(rpcvers=3)); L3[58] = 1
    assert status_of(bytes(L3)) == O.E_RPC
    # cred pad bytes are checked too (strict)
    L4 = bytearray(call_logical(cred=(1, b"xy"))); L4[34] = 9  # cred body 32..34, pad 34..36
    assert status_of(bytes(L4)) == O.E_PAD


def test_status_codes_items():
    cfg = O.Config(prog=CFG.prog, vers=CFG.vers, user_schemas={40: [O.K_I32_VAR, O.K_F64_VAR]})
    a = np.arange(5, dtype=np.int32)
    L = O.call_header(1, cfg.prog, cfg.vers, 40) + O.put_array(a) + O.put_array(np.zeros(2, np.float64))
    c = O.parse_call(L, cfg)
    assert c.status == O.OK
    assert O.decode_item(L, c, 0, O.K_I32_VAR, 5)[0] == O.OK
    assert O.decode_item(L, c, 0, O.K_I32_VAR, 4)[0] == O.E_SIZE
    assert O.decode_item(L, c, 0, O.K_U32_VAR, 5)[0] == O.E_ARG
    assert O.decode_item(L, c, 2, O.K_I32_VAR, 5)[0] == O.E_ARG
    Lbad = L[:-1]
    assert O.parse_call(Lbad, cfg).status == O.E_TRUNCATED


def test_scan_status_codes():
    w1 = O.frame(call_logical(xid=1), 16)
    w2 = O.frame(call_logical(xid=2), 16)
    ring = ring_of(w1 + w2, 512)
    full = len(w1) + len(w2)
    s = O.frame_scan(ring, 0, full)
    assert s.status == O.OK and s.consumed == full and len(s.recs) == 2
    for t in range(full):  # every truncation: INCOMPLETE, consumed at the last record boundary
        s = O.frame_scan(ring, 0, t)
        want = 0 if t < len(w1) else len(w1)
        assert s.consumed == want
        assert s.status == (O.OK if t in (0, len(w1)) else O.INCOMPLETE)
    s = O.frame_scan(ring, 0, full, max_record_bytes=len(call_logical()) - 1)
    assert s.status == O.E_FRAG and s.consumed == 0
    s = O.frame_scan(ring, 0, full, max_frags=len(w1) // 20)
    assert s.status == O.E_CAPACITY and s.consumed == 0 and s.recs == []
    n1 = O.frame_count(len(call_logical()), 16)
    s = O.frame_scan(ring, 0, full, max_frags=n1 + 1)
    assert s.status == O.INCOMPLETE and s.consumed == len(w1) and len(s.recs) == 1 and len(s.frags) == n1
    s = O.frame_scan(ring, 0, full, max_records=1)
    assert s.status == O.INCOMPLETE and s.consumed == len(w1)
    # E_FRAG on the header, before the data has arrived (reading R8)
    big = hdr(0x7FFFFFF0, True)
    s = O.frame_scan(ring_of(big, 64), 0, 4, max_record_bytes=1 << 20)
    assert s.status == O.E_FRAG


def test_scan_consumed_monotone_and_invariants():
    calls = [call_logical(xid=i, data=bytes(range(i * 7 % 50))) for i in range(12)]
    wire = b"".join(O.frame(L, 8 + 4 * (i % 5)) for i, L in enumerate(calls))
    ring = ring_of(wire, 4096)
    prev = 0
    for t in range(0, len(wire) + 1, 7):
        s = O.frame_scan(ring, 0, t)
        assert s.consumed >= prev
        prev = s.consumed
        for r in s.recs:
            fr = s.frags[r["frag0"]:r["frag0"] + r["nfrags"]]
            assert sum(f["len"] for f in fr) == r["len"]
            assert [f["last"] for f in fr].count(1) == 1 and fr[-1]["last"] == 1


def test_serve_statuses_and_replies():
    region = np.zeros(1 << 16, np.uint8)
    base = 0x7F0000000000
    src = gen.random_bytes(3, 3000)
    region[20000:23000] = src
    recs = [
        O.encode_call(10, gen.PROC_H2D, [(O.K_U64, base + 100), (O.K_OPAQUE_VAR, b"hello"), (O.K_U64, 5)], CFG),
        O.encode_call(11, gen.PROC_D2H, [(O.K_U64, base + 20000), (O.K_U64, 3000)], CFG, F=1024),
        O.encode_call(10, gen.PROC_H2D, [(O.K_U64, base + 200), (O.K_OPAQUE_VAR, b"dup"), (O.K_U64, 3)], CFG),
        O.encode_call(12, gen.PROC_H2D, [(O.K_U64, base + (1 << 16) - 2), (O.K_OPAQUE_VAR, b"xyz"), (O.K_U64, 3)],
                      CFG),
        O.encode_call(13, gen.PROC_D2H, [(O.K_U64, base - 1), (O.K_U64, 4)], CFG),
        O.frame(call_logical(xid=14, mtype=1), 64),
    ]
    wire = b"".join(recs)
    out = O.serve([(ring_of(wire, 8192), 0, len(wire))], O.Config(**{**CFG.__dict__, "frag_payload": 1024}),
                  region, base, [1 << 14], [0])
    st_ = [r["status"] for r in out["records"]]
    assert st_ == [O.OK, O.OK, O.E_XID, O.E_PTR, O.E_PTR, O.E_RPC]
    assert [r["reply_err"] for r in out["records"]] == [0, 0, -1, 1, 1, -1]
    assert bytes(region[100:105]) == b"hello" and region[200] == 0
    send = out["send"][0]
    r0 = out["records"][0]
    assert bytes(send[:r0["reply_wire"]]) == O.frame(O.reply_header(10) + O.put_u32(0), 1024)
    r1 = out["records"][1]
    assert bytes(send[r1["reply_off"]:r1["reply_off"] + r1["reply_wire"]]) == O.encode_memcpy_d2h(11, src, 0, 1024)
    r4 = out["records"][4]
    assert bytes(send[r4["reply_off"]:r4["reply_off"] + r4["reply_wire"]]) == O.frame(
        O.reply_header(13) + O.put_u32(1), 1024)
    assert out["reply_bytes"][0] == sum(r["reply_wire"] for r in out["records"])


# ------------------------------------------------------------------ round trips

item_strategy = st.one_of(
    st.tuples(st.just(O.K_U32), st.integers(0, 2**32 - 1)),
    st.tuples(st.just(O.K_U64), st.integers(0, 2**64 - 1)),
    st.tuples(st.just(O.K_OPAQUE_VAR), st.binary(max_size=300)),
    st.tuples(st.sampled_from([O.K_I32_VAR, O.K_U32_VAR, O.K_F32_VAR, O.K_I64_VAR, O.K_U64_VAR, O.K_F64_VAR]),
              st.integers(0, 100), st.integers(0, 2**31)),
)


@settings(max_examples=150, deadline=None)
@given(st.lists(item_strategy, min_size=1, max_size=8), st.integers(1, 400), st.integers(0, 3000))
def test_round_trip_decode_encode(items, F, at):
    kinds, vals = [], []
    for it in items:
        if it[0] in (O.K_U32, O.K_U64, O.K_OPAQUE_VAR):
            kinds.append(it[0]); vals.append(it[1])
        else:
            dt = gen.NP_DTYPE[it[0]]
            kinds.append(it[0]); vals.append(gen.random_elems(gen.rng(it[2]), dt, it[1]))
    cfg = O.Config(prog=CFG.prog, vers=CFG.vers, user_schemas={50: kinds})
    w = O.encode_call(77, 50, list(zip(kinds, vals)), cfg, F=F)
    # 8 KiB ring so most cases wrap; F=1 framing of a large record can exceed it (5 wire B per logical B)
    ring = ring_of(w, 1 << 13 if len(w) <= 1 << 13 else None, at)
    s = O.frame_scan(ring, at, at + len(w))
    assert s.status == O.OK and len(s.recs) == 1
    L = O.record_logical(ring, s, 0)
    c = O.parse_call(L, cfg)
    assert c.status == O.OK and c.end == len(L)
    for i, (k, v) in enumerate(zip(kinds, vals)):
        if k in (O.K_U32, O.K_U64):
            assert c.value[i] == v
        elif k == O.K_OPAQUE_VAR:
            stt, out = O.decode_item(L, c, i, k, len(v))
            assert stt == O.OK and out.tobytes() == v
            assert all(b == 0 for b in L[c.off[i] + len(v):c.off[i] + len(v) + (-len(v)) % 4])
        else:
            stt, out = O.decode_item(L, c, i, k, len(v))
            assert stt == O.OK and out.tobytes() == v.tobytes()
    # encode(decode(w)) == w for canonical w (greedy framing, zero pads)
    dec = []
    for i, (k, v) in enumerate(zip(kinds, vals)):
        if k in (O.K_U32, O.K_U64):
            dec.append((k, int(c.value[i])))
        else:
            stt, out = O.decode_item(L, c, i, k, c.count[i])
            dec.append((k, out if k == O.K_OPAQUE_VAR else out.view(gen.NP_DTYPE[k])))
    assert O.encode_call(77, 50, dec, cfg, F=F) == w


@settings(max_examples=60, deadline=None)
@given(st.binary(max_size=5000), st.integers(1, 9000), st.sampled_from([0, 1, 2, 3]))
def test_d2h_reply_round_trip(data, F, err):
    F = F * 4 if F % 3 == 0 else F
    w = O.encode_memcpy_d2h(0x99, data, 1 if err == 3 else 0, F)
    ring = ring_of(w, 1 << 15)
    s = O.frame_scan(ring, 0, len(w))
    assert s.status == O.OK and len(s.recs) == 1
    L = O.record_logical(ring, s, 0)
    assert L[:24] == O.reply_header(0x99)
    if err == 3:
        assert L[24:] == O.put_u32(1)
    else:
        up = xdrlib.Unpacker(L[24:])
        assert up.unpack_int() == 0 and up.unpack_opaque() == data
        up.done()
    fl = [f["len"] for f in s.frags]
    assert all(x == F for x in fl[:-1]) and 0 < fl[-1] <= F or (len(L) == 0)


def test_array_reply_vs_xdrlib():
    """or_encode_array_reply (used as the expected value of the GPU typed-array encoder) decoded by xdrlib."""
    for dt, unpack in ((np.int32, "unpack_int"), (np.uint32, "unpack_uint"), (np.int64, "unpack_hyper"),
                       (np.uint64, "unpack_uhyper")):
        a = gen.random_elems(gen.rng(7), dt, 3001)
        for F in (97, 4096, 65536):
            w = O.encode_array_reply(0xABCD, a, 0, F)
            ring = ring_of(w, 1 << 16)
            s = O.frame_scan(ring, 0, len(w))
            assert s.status == O.OK and all(f["len"] == F for f in s.frags[:-1])
            L = O.record_logical(ring, s, 0)
            up = xdrlib.Unpacker(L)
            assert [up.unpack_uint() for _ in range(6)] == [0xABCD, 1, 0, 0, 0, 0]
            assert up.unpack_int() == 0
            assert up.unpack_array(getattr(up, unpack)) == [int(x) for x in a]
            up.done()
    w = O.encode_array_reply(5, np.zeros(3, np.float64), 1, 4096)
    assert w == struct.pack(">I", 0x80000000 | 28) + O.reply_header(5) + struct.pack(">i", 1)


@given(st.binary(min_size=0, max_size=300), st.lists(st.integers(0, 40), min_size=0, max_size=12))
def test_frame_lens_vs_hand_framing(L, cuts):
    """or_frame_record_lens against record marks written with struct (RFC 5531 §11)."""
    lens, left = [], len(L)
    for c in cuts:
        c = min(c, left)
        lens.append(c)
        left -= c
    lens.append(left)
    want, o = b"", 0
    for i, n in enumerate(lens):
        want += struct.pack(">I", n | (0x80000000 if i == len(lens) - 1 else 0)) + L[o:o + n]
        o += n
    assert O.frame_lens(L, lens) == want


def test_serve_lenient_mode():
    """Lenient serve (readings R5, R9): nonzero pads and trailing bytes pass, HtoD copies min(n, size)."""
    lenient = O.Config(prog=CFG.prog, vers=CFG.vers, strict=False, proc_h2d=CFG.proc_h2d, proc_d2h=CFG.proc_d2h)
    region = np.zeros(4096, np.uint8)
    base = 0x10000
    L1 = bytearray(call_logical(xid=1, data=b"abcde", size=3))       # n=5, size=3 -> copies 3
    L1[20:24] = struct.pack(">I", CFG.proc_h2d)
    L1[36:40] = struct.pack(">I", 0)
    L1[40:48] = struct.pack(">Q", base + 100)
    L2 = bytearray(call_logical(xid=2, data=b"xyz", extra=b"\0\0\0\0"))  # trailing bytes ignored
    L2[40:48] = struct.pack(">Q", base + 200)
    L2[52 + 3] = 9                                                       # nonzero pad ignored
    wire = O.frame(bytes(L1), 64) + O.frame(bytes(L2), 64)
    out = O.serve([(ring_of(wire, 4096), 0, len(wire))], lenient, region, base, [1 << 12], [0])
    assert [r["status"] for r in out["records"]] == [O.OK, O.OK]
    assert bytes(region[100:106]) == b"abc\0\0\0" and bytes(region[200:203]) == b"xyz"
    strict = O.serve([(ring_of(wire, 4096), 0, len(wire))], CFG, np.zeros(4096, np.uint8), base, [1 << 12], [0])
    assert [r["status"] for r in strict["records"]] == [O.E_SIZE, O.E_PAD]


def test_reply_item_vs_xdrlib():
    """or_encode_reply_item (expected value of the GPU batched reply encoder) decoded by xdrlib."""
    cases = [(O.K_U32, 0xDEADBEEF, None, "unpack_uint"), (O.K_U64, 0x0123456789ABCDEF, None, "unpack_uhyper"),
             (O.K_OPAQUE_VAR, 0, gen.random_bytes(1, 13), "unpack_opaque"),
             (O.K_I64_VAR, 0, gen.random_elems(gen.rng(2), np.int64, 9), "hyper_array"),
             (O.K_F32_FIX, 0, np.arange(5, dtype=np.float32), "float_farray")]
    for kind, value, elems, how in cases:
        w = O.encode_reply_item(7, 0, kind, value, elems, 4096)
        L = w[4:]
        assert struct.unpack(">I", w[:4])[0] == 0x80000000 | len(L)
        up = xdrlib.Unpacker(L)
        assert [up.unpack_uint() for _ in range(6)] == [7, 1, 0, 0, 0, 0] and up.unpack_int() == 0
        if how == "unpack_uint":
            assert up.unpack_uint() == value
        elif how == "unpack_uhyper":
            assert up.unpack_uhyper() == value
        elif how == "unpack_opaque":
            assert up.unpack_opaque() == elems.tobytes()
        elif how == "hyper_array":
            assert up.unpack_array(up.unpack_hyper) == [int(x) for x in elems]
        else:
            assert up.unpack_farray(5, up.unpack_float) == [float(x) for x in elems]
        up.done()
    assert O.encode_reply_item(9, 35, O.K_U64, 5) == struct.pack(">I", 0x80000000 | 28) + O.reply_header(9) + \
        struct.pack(">i", 35)
