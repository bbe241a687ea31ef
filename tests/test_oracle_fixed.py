"""Pins the oracle's fixed-length XDR kinds (RFC 4506 §4.9 fixed-length opaque `opaque[n]`, §4.12
fixed-length array `T[n]`; PAPER.md:144 names ONC RPC / XDR as the wire format) to Python's xdrlib,
an independent encoder/decoder.  CPU only.

The branch under test is or_parse_call's `cnt = fixed` (no count word on the wire) and the pad after
`opaque[n]`, plus or_decode_item for the *_FIX kinds.  Every expected offset, count and value below
comes from xdrlib (`Packer.pack_fopaque` / `pack_farray`, `Unpacker.unpack_fopaque` / `unpack_farray`)
or from numpy big-endian views, never from the oracle.  A plausible mistake -- reading a count word for
`T[n]`, skipping `opaque[13]`'s 3-byte pad, taking the pad for 4/8-byte elements, swapping 8-byte
halves -- moves an offset or a value and fails here.
"""
import struct
import warnings

import numpy as np
import pytest

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import gen

with warnings.catch_warnings():
    warnings.simplefilter("ignore", DeprecationWarning)
    import xdrlib

PROC = 41
FIX = {O.K_I32_FIX: (np.int32, "I"), O.K_U32_FIX: (np.uint32, "I"), O.K_F32_FIX: (np.float32, "I"),
       O.K_I64_FIX: (np.int64, "Q"), O.K_U64_FIX: (np.uint64, "Q"), O.K_F64_FIX: (np.float64, "Q")}


def packer_with_header(xid: int, proc: int) -> xdrlib.Packer:
    """CALL header (RFC 5531 §9: xid, CALL, rpcvers 2, prog, vers, proc, AUTH_NONE cred and verf) by xdrlib."""
    p = xdrlib.Packer()
    for v in (xid, 0, 2, gen.PROG, gen.VERS, proc, 0):
        p.pack_uint(v)
    p.pack_opaque(b"")
    p.pack_uint(0)
    p.pack_opaque(b"")
    return p


def pack_fixed(p: xdrlib.Packer, kind: int, value):
    if kind == O.K_OPAQUE_FIX:
        p.pack_fopaque(len(value), bytes(value))
        return
    dt, code = FIX[kind]
    u = np.asarray(value, dt).view(np.uint32 if code == "I" else np.uint64)
    p.pack_farray(len(u), [int(x) for x in u], p.pack_uint if code == "I" else p.pack_uhyper)


def build(items):
    """items: [(kind, value)] -> (schema codes, logical record, xdrlib offset of every item's data)."""
    p = packer_with_header(0x0F1F0F1F, PROC)
    codes, offs = [], []
    for kind, value in items:
        codes.append(O.item_code(kind, len(value)))
        offs.append(len(p.get_buffer()))  # fixed kinds: the data starts where the item starts
        pack_fixed(p, kind, value)
    return codes, p.get_buffer(), offs


def elems(kind, n, seed):
    return gen.random_elems(gen.rng(seed), FIX[kind][0], n)


# every fixed kind once, odd opaque lengths (pads 3, 2, 1, 0), ragged element counts
CASES = [
    [(O.K_OPAQUE_FIX, np.arange(13, dtype=np.uint8))],
    [(O.K_OPAQUE_FIX, np.arange(1, 3, dtype=np.uint8)), (O.K_I32_FIX, elems(O.K_I32_FIX, 7, 1))],
    [(O.K_U32_FIX, elems(O.K_U32_FIX, 3, 2)), (O.K_OPAQUE_FIX, np.full(7, 0xAB, np.uint8)),
     (O.K_F32_FIX, elems(O.K_F32_FIX, 11, 3))],
    [(O.K_I64_FIX, elems(O.K_I64_FIX, 2, 4)), (O.K_OPAQUE_FIX, np.arange(8, dtype=np.uint8)),
     (O.K_U64_FIX, elems(O.K_U64_FIX, 5, 5)), (O.K_F64_FIX, elems(O.K_F64_FIX, 11, 6))],
    [(O.K_OPAQUE_FIX, np.arange(1, dtype=np.uint8)), (O.K_F64_FIX, elems(O.K_F64_FIX, 1, 7)),
     (O.K_OPAQUE_FIX, np.arange(5, dtype=np.uint8)), (O.K_I32_FIX, elems(O.K_I32_FIX, 1, 8)),
     (O.K_OPAQUE_FIX, np.arange(6, dtype=np.uint8)), (O.K_U32_FIX, elems(O.K_U32_FIX, 2, 9)),
     (O.K_OPAQUE_FIX, np.arange(3, dtype=np.uint8)), (O.K_I64_FIX, elems(O.K_I64_FIX, 3, 10))],
]


@pytest.mark.parametrize("items", CASES, ids=[f"case{i}" for i in range(len(CASES))])
def test_fixed_kinds_parse_and_decode_vs_xdrlib(items):
    codes, L, offs = build(items)
    cfg = O.Config(prog=gen.PROG, vers=gen.VERS, user_schemas={PROC: codes})
    c = O.parse_call(L, cfg)
    assert c.status == O.OK and c.n_items == len(items)
    assert c.end == len(L)  # the whole record consumed: no count word read, every pad skipped
    up = xdrlib.Unpacker(L[40:])
    for i, (kind, value) in enumerate(items):
        n = len(value)
        assert c.kind[i] == kind
        assert c.off[i] == offs[i], (i, kind)
        assert c.count[i] == n
        st, out = O.decode_item(L, c, i, kind, n)
        assert st == O.OK
        if kind == O.K_OPAQUE_FIX:
            ref = up.unpack_fopaque(n)  # xdrlib reads the data and skips the pad
            assert out.tobytes() == ref == bytes(value)
            continue
        dt, code = FIX[kind]
        ref = up.unpack_farray(n, up.unpack_uint if code == "I" else up.unpack_uhyper)
        got = out.view(np.uint32 if code == "I" else np.uint64)
        assert [int(x) for x in got] == ref
        be = np.frombuffer(L, dtype=">u4" if code == "I" else ">u8", count=n, offset=offs[i])
        assert np.array_equal(got, be)
        assert out.tobytes() == np.asarray(value, dt).tobytes()  # bit-exact (reading R13)
    up.done()  # xdrlib agrees that nothing trails the last item


def test_fixed_opaque_pad_is_checked():
    """opaque[13] carries 3 zero pad bytes (RFC 4506 §4.9); strict mode rejects a nonzero one (reading R5)."""
    items = [(O.K_OPAQUE_FIX, np.arange(13, dtype=np.uint8)), (O.K_I32_FIX, np.arange(2, dtype=np.int32))]
    codes, L, offs = build(items)
    strict = O.Config(prog=gen.PROG, vers=gen.VERS, user_schemas={PROC: codes})
    lenient = O.Config(prog=gen.PROG, vers=gen.VERS, strict=False, user_schemas={PROC: codes})
    assert offs[1] == offs[0] + 16  # xdrlib: 13 data bytes + 3 pad
    for k in range(3):
        bad = bytearray(L)
        bad[offs[0] + 13 + k] = 0x5A
        assert O.parse_call(bytes(bad), strict).status == O.E_PAD
        c = O.parse_call(bytes(bad), lenient)
        assert c.status == O.OK and c.off[1] == offs[1]


def test_fixed_kinds_truncation_and_no_count_word():
    items = [(O.K_I32_FIX, np.arange(4, dtype=np.int32))]
    codes, L, _ = build(items)
    cfg = O.Config(prog=gen.PROG, vers=gen.VERS, user_schemas={PROC: codes})
    assert O.parse_call(L[:-1], cfg).status == O.E_TRUNCATED
    # the same bytes with a count word in front are one word too long for int[4]: strict E_TRAILING
    p = packer_with_header(0x0F1F0F1F, PROC)
    p.pack_array([0, 1, 2, 3], p.pack_int)
    assert O.parse_call(p.get_buffer(), cfg).status == O.E_TRAILING
    # ... and as int<> they parse (the VAR kind reads the count word)
    var = O.Config(prog=gen.PROG, vers=gen.VERS, user_schemas={PROC: [O.K_I32_VAR]})
    c = O.parse_call(p.get_buffer(), var)
    assert c.status == O.OK and c.count[0] == 4 and c.off[0] == 44
    # opaque[0] and T[0]: no bytes at all
    codes0 = [O.item_code(O.K_OPAQUE_FIX, 0), O.item_code(O.K_F64_FIX, 0), O.K_U32]
    p = packer_with_header(0x0F1F0F1F, PROC)
    p.pack_uint(0xDEADBEEF)
    c = O.parse_call(p.get_buffer(), O.Config(prog=gen.PROG, vers=gen.VERS, user_schemas={PROC: codes0}))
    assert c.status == O.OK and c.off[0] == 40 and c.off[1] == 40 and c.value[2] == 0xDEADBEEF
    assert struct.unpack(">I", p.get_buffer()[40:44])[0] == 0xDEADBEEF


def test_d2h_size_beyond_opaque_length_is_eptr():
    """DESIGN.md reading R21: opaque<>'s length word is an unsigned int (RFC 4506 §4.10, at most 2^32 - 1
    bytes), so a memcpy DtoH CALL asking for size >= 2^32 cannot be answered with data even when the whole
    range lies inside the registered region: E_PTR and the void arm (reply err = 1), like any DtoH the
    server cannot serve.  The region is a lazily allocated 4 GiB + 4 KiB of zeros (never touched)."""
    cfg = O.Config(prog=gen.PROG, vers=gen.VERS, frag_payload=4096)
    region = np.zeros((1 << 32) + 4096, np.uint8)  # calloc: no pages are touched
    base = 1 << 44
    wire = (O.encode_call(21, gen.PROC_D2H, [(O.K_U64, base), (O.K_U64, 1 << 32)], cfg)
            + O.encode_call(22, gen.PROC_D2H, [(O.K_U64, base + 8), (O.K_U64, 16)], cfg))
    ring = np.zeros(1 << 9, np.uint8)
    ring[:len(wire)] = np.frombuffer(wire, np.uint8)
    out = O.serve([(ring, 0, len(wire))], cfg, region, base, [1 << 12], [0])
    assert [r["status"] for r in out["records"]] == [O.E_PTR, O.OK]
    assert [r["reply_err"] for r in out["records"]] == [1, 0]
    # the void-arm reply: REPLY header (24 B) + err = 1, one fragment -- spelled out with xdrlib
    p = xdrlib.Packer()
    for v in (21, 1, 0, 0, 0, 0, 1):
        p.pack_uint(v)
    L = p.get_buffer()
    want = struct.pack(">I", 0x80000000 | len(L)) + L
    r0 = out["records"][0]
    assert bytes(out["send"][0][r0["reply_off"]:r0["reply_off"] + r0["reply_wire"]]) == want
