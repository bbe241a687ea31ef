"""Pins the oracle against glibc's Sun-RPC XDR implementation (a third-party encoder/decoder).

glibc 2.39 keeps the Sun RPC routines as compat symbols only (version GLIBC_2.2.5), so they are looked
up with dlvsym.  Layouts below are the x86-64 ones of <rpc/xdr.h> / <rpc/rpc_msg.h>.
Covers: RFC 5531 §9 CALL/REPLY headers (xdr_callmsg / xdr_replymsg), RFC 4506 §4.5 hyper order
(xdr_u_hyper), §4.10 opaque padding (xdr_bytes), §4.6/4.7 float/double bits, and RFC 5531 §11 record
marking in both directions (xdrrec_*).  Known disagreement (reading R1): glibc rejects a
zero-length non-last fragment, which RFC 5531 §11 permits, so that case is pinned by brute force in
test_oracle_pins.py instead.
"""
import ctypes as C
import struct
import warnings

import numpy as np
import pytest

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import gen

libc = C.CDLL("libc.so.6")
_dlvsym = libc.dlvsym
_dlvsym.restype = C.c_void_p
_dlvsym.argtypes = [C.c_void_p, C.c_char_p, C.c_char_p]


def sym(name, restype, *argtypes):
    addr = _dlvsym(libc._handle, name.encode(), b"GLIBC_2.2.5")
    if not addr:
        pytest.skip(f"glibc compat symbol {name} not available")
    return C.CFUNCTYPE(restype, *argtypes)(addr)


class XDR(C.Structure):
    _fields_ = [("x_op", C.c_int), ("x_ops", C.c_void_p), ("x_public", C.c_void_p), ("x_private", C.c_void_p),
                ("x_base", C.c_void_p), ("x_handy", C.c_uint)]


class OpaqueAuth(C.Structure):
    _fields_ = [("oa_flavor", C.c_int), ("oa_base", C.c_void_p), ("oa_length", C.c_uint)]


class CallBody(C.Structure):
    _fields_ = [("cb_rpcvers", C.c_ulong), ("cb_prog", C.c_ulong), ("cb_vers", C.c_ulong), ("cb_proc", C.c_ulong),
                ("cb_cred", OpaqueAuth), ("cb_verf", OpaqueAuth)]


class ARResults(C.Structure):
    _fields_ = [("where", C.c_void_p), ("proc", C.c_void_p)]


class AcceptedReply(C.Structure):
    _fields_ = [("ar_verf", OpaqueAuth), ("ar_stat", C.c_int), ("ar_results", ARResults)]


class ReplyBody(C.Structure):
    _fields_ = [("rp_stat", C.c_int), ("rp_acpt", AcceptedReply)]


class MsgBody(C.Union):
    _fields_ = [("cmb", CallBody), ("rmb", ReplyBody)]


class RpcMsg(C.Structure):
    _fields_ = [("rm_xid", C.c_ulong), ("rm_direction", C.c_int), ("ru", MsgBody)]


XDR_ENCODE, XDR_DECODE = 0, 1
xdrmem_create = sym("xdrmem_create", None, C.POINTER(XDR), C.c_void_p, C.c_uint, C.c_int)
xdr_callmsg = sym("xdr_callmsg", C.c_int, C.POINTER(XDR), C.POINTER(RpcMsg))
xdr_replymsg = sym("xdr_replymsg", C.c_int, C.POINTER(XDR), C.POINTER(RpcMsg))
xdr_u_hyper = sym("xdr_u_hyper", C.c_int, C.POINTER(XDR), C.POINTER(C.c_uint64))
xdr_bytes = sym("xdr_bytes", C.c_int, C.POINTER(XDR), C.POINTER(C.c_void_p), C.POINTER(C.c_uint), C.c_uint)
xdr_float = sym("xdr_float", C.c_int, C.POINTER(XDR), C.POINTER(C.c_float))
xdr_double = sym("xdr_double", C.c_int, C.POINTER(XDR), C.POINTER(C.c_double))
xdr_int = sym("xdr_int", C.c_int, C.POINTER(XDR), C.POINTER(C.c_int))
xdr_opaque = sym("xdr_opaque", C.c_int, C.POINTER(XDR), C.c_void_p, C.c_uint)
XDR_VOID_ADDR = _dlvsym(libc._handle, b"xdr_void", b"GLIBC_2.2.5")
RW = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_void_p, C.c_int)
xdrrec_create = sym("xdrrec_create", None, C.POINTER(XDR), C.c_uint, C.c_uint, C.c_void_p, RW, RW)
xdrrec_endofrecord = sym("xdrrec_endofrecord", C.c_int, C.POINTER(XDR), C.c_int)
xdrrec_skiprecord = sym("xdrrec_skiprecord", C.c_int, C.POINTER(XDR))


def mem_encode(fn, *args, size=4096):
    buf = C.create_string_buffer(size)
    x = XDR()
    xdrmem_create(C.byref(x), C.addressof(buf), size, XDR_ENCODE)
    assert fn(C.byref(x), *args)
    return buf.raw[: size - x.x_handy]


def test_callmsg_matches_oracle_and_golden(golden_dir):
    m = RpcMsg()
    m.rm_xid = 0x12345678
    m.rm_direction = 0
    m.ru.cmb.cb_rpcvers, m.ru.cmb.cb_prog, m.ru.cmb.cb_vers, m.ru.cmb.cb_proc = 2, 99, 1, 440
    g = mem_encode(xdr_callmsg, C.byref(m))
    assert len(g) == 40
    assert O.call_header(0x12345678, 99, 1, 440) == g
    gold = {ln.split()[0]: bytes.fromhex("".join(ln.split()[1:]))
            for ln in open(f"{golden_dir}/rfc5531_call_reply_headers.txt") if ln.strip() and ln[0] != "#"}
    assert gold["call"] == g


def test_callmsg_with_auth_bodies():
    # cred/verf bodies of length 0..9 (pad 0..3): glibc writes opaque_auth exactly as RFC 5531 §8.2
    for cl in range(10):
        for vl in (0, 3, 8):
            cb = bytes((7 * i + 1) & 0xFF for i in range(cl))
            vb = bytes((5 * i + 3) & 0xFF for i in range(vl))
            cbuf, vbuf = C.create_string_buffer(cb, max(1, cl)), C.create_string_buffer(vb, max(1, vl))
            m = RpcMsg()
            m.rm_xid, m.rm_direction = 0xDEADBEEF, 0
            m.ru.cmb.cb_rpcvers, m.ru.cmb.cb_prog, m.ru.cmb.cb_vers, m.ru.cmb.cb_proc = 2, 0x20000099, 3, 17
            m.ru.cmb.cb_cred = OpaqueAuth(1, C.addressof(cbuf), cl)
            m.ru.cmb.cb_verf = OpaqueAuth(6, C.addressof(vbuf), vl)
            g = mem_encode(xdr_callmsg, C.byref(m))
            assert O.call_header(0xDEADBEEF, 0x20000099, 3, 17, (1, cb), (6, vb)) == g


def test_replymsg_matches_oracle():
    m = RpcMsg()
    m.rm_xid, m.rm_direction = 0x12345678, 1
    m.ru.rmb.rp_stat = 0
    m.ru.rmb.rp_acpt.ar_stat = 0
    m.ru.rmb.rp_acpt.ar_results.proc = XDR_VOID_ADDR
    g = mem_encode(xdr_replymsg, C.byref(m))
    assert len(g) == 24
    assert O.reply_header(0x12345678) == g


@pytest.mark.parametrize("v", [0x00007F0000001000, 0, 1, 0xFFFFFFFFFFFFFFFF, 0x0123456789ABCDEF, 1 << 63])
def test_u_hyper(v):
    x = C.c_uint64(v)
    assert O.put_u64(v) == mem_encode(xdr_u_hyper, C.byref(x))


@pytest.mark.parametrize("n", list(range(0, 13)) + [4093, 4096])
def test_xdr_bytes_padding(n):
    data = bytes((i * 31 + 7) & 0xFF for i in range(n))
    buf = C.create_string_buffer(data, max(1, n))
    p = C.c_void_p(C.addressof(buf))
    ln = C.c_uint(n)
    g = mem_encode(xdr_bytes, C.byref(p), C.byref(ln), 1 << 20, size=n + 64)
    assert O.put_opaque_var(data) == g


def test_float_double_bits():
    f32 = gen.special_bits(np.float32)
    f64 = gen.special_bits(np.float64)
    for v in f32:
        g = mem_encode(xdr_float, C.byref(C.c_float.from_buffer_copy(v.tobytes())))
        assert O.put_array(np.array([v], np.float32), with_count=False) == g
    for v in f64:
        g = mem_encode(xdr_double, C.byref(C.c_double.from_buffer_copy(v.tobytes())))
        assert O.put_array(np.array([v], np.float64), with_count=False) == g
    for v in (-(1 << 31), -1, 0, 1, (1 << 31) - 1):
        assert O.put_array(np.array([v], np.int32), with_count=False) == mem_encode(xdr_int, C.byref(C.c_int(v)))


def glibc_frame(logical: bytes, sendsize: int) -> bytes:
    """Writes `logical` (multiple of 4) as one record through xdrrec with the given sendsize."""
    out = bytearray()

    def writeit(h, buf, n):
        out.extend(C.string_at(buf, n))
        return n

    def readit(h, buf, n):
        return -1

    w, r = RW(writeit), RW(readit)
    x = XDR()
    xdrrec_create(C.byref(x), sendsize, sendsize, None, r, w)
    x.x_op = XDR_ENCODE
    b = C.create_string_buffer(logical, max(1, len(logical)))
    # xdr_opaque writes the bytes plus pad; logical is a multiple of 4, so it adds nothing
    step = 1 << 16
    for o in range(0, len(logical), step):
        chunk = logical[o:o + step]
        cb = C.create_string_buffer(chunk, len(chunk))
        assert xdr_opaque(C.byref(x), C.addressof(cb), len(chunk))
    assert xdrrec_endofrecord(C.byref(x), 1)
    del b
    return bytes(out)


def glibc_read_record(wire: bytes, nbytes: int) -> bytes:
    pos = [0]

    def readit(h, buf, n):
        k = min(n, len(wire) - pos[0])
        if k <= 0:
            return -1
        C.memmove(buf, wire[pos[0]:pos[0] + k], k)
        pos[0] += k
        return k

    def writeit(h, buf, n):
        return -1

    w, r = RW(writeit), RW(readit)
    x = XDR()
    xdrrec_create(C.byref(x), 4000, 4000, None, r, w)
    x.x_op = XDR_DECODE
    assert xdrrec_skiprecord(C.byref(x))
    out = C.create_string_buffer(max(1, nbytes))
    ok = xdr_opaque(C.byref(x), C.addressof(out), nbytes)
    return out.raw[:nbytes] if ok else None


@pytest.mark.parametrize("F", [100, 3996, 65536])
@pytest.mark.parametrize("n", [4, 96, 100, 104, 200, 3996, 4000, 65536, 65540, 200000])
def test_xdrrec_encode_matches_oracle_framing(F, n):
    if n % 4:
        pytest.skip("xdrrec records are built from 4-byte XDR units")
    L = gen.random_bytes(n * 7 + F, n).tobytes()
    assert glibc_frame(L, F + 4) == O.frame(L, F)
    # closed form: wire = n + 4 * max(1, ceil(n / F))
    assert len(O.frame(L, F)) == n + 4 * max(1, -(-n // F))


def test_xdrrec_decode_agrees_with_oracle_scan():
    g = gen.rng(1234)
    for trial in range(60):
        n = int(g.integers(1, 600)) * 4
        L = gen.random_bytes(trial, n).tobytes()
        k = int(g.integers(1, 8))
        cuts = sorted(set(int(c) for c in g.integers(1, n, size=k - 1))) if n > 1 and k > 1 else []
        lens = [b - a for a, b in zip([0] + cuts, cuts + [n])]
        wire = b"".join(struct.pack(">I", ln | ((i == len(lens) - 1) << 31)) + L[sum(lens[:i]):sum(lens[:i + 1])]
                        for i, ln in enumerate(lens))
        assert glibc_read_record(wire, n) == L
        ring = np.zeros(1 << 12, np.uint8)
        ring[: len(wire)] = np.frombuffer(wire, np.uint8)
        s = O.frame_scan(ring, 0, len(wire))
        assert s.status == O.OK and len(s.recs) == 1
        assert O.record_logical(ring, s, 0) == L
        assert [f["len"] for f in s.frags] == lens


def test_glibc_rejects_zero_length_nonlast_fragment_but_oracle_accepts():
    """Reading R1: RFC 5531 §11 allows fragment lengths 0..2^31-1; glibc refuses header 0x00000000."""
    L = b"ABCDEFGH"
    wire = struct.pack(">I", 0) + struct.pack(">I", 0x80000000 | 8) + L
    assert glibc_read_record(wire, 8) is None
    ring = np.zeros(64, np.uint8)
    ring[: len(wire)] = np.frombuffer(wire, np.uint8)
    s = O.frame_scan(ring, 0, len(wire))
    assert s.status == O.OK and O.record_logical(ring, s, 0) == L


def test_glibc_accepts_trailing_empty_last_fragment():
    L = b"ABCDEFGH"
    wire = struct.pack(">I", 8) + L + struct.pack(">I", 0x80000000)
    assert glibc_read_record(wire, 8) == L
    ring = np.zeros(64, np.uint8)
    ring[: len(wire)] = np.frombuffer(wire, np.uint8)
    s = O.frame_scan(ring, 0, len(wire))
    assert s.status == O.OK and O.record_logical(ring, s, 0) == L and len(s.frags) == 2
