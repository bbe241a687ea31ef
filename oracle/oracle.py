"""ORACLE — TEST INFRASTRUCTURE ONLY.

ctypes marshalling around ``oracle/oracle.c`` (the plain byte-at-a-time CPU implementation of RFC 5531
record marking / CALL-REPLY headers and RFC 4506 XDR, see its header for the citations).  Argument
conversion only: every step of the computation is in the C file.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` / ``--impl reference``
legs may import this module.  It imports nothing from the CUDA package and the CUDA package imports
nothing from here.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "oracle.c")
LIBPATH = os.path.join(HERE, "liboracle.so")

# status codes, restated independently of include/crk.h
OK, INCOMPLETE = 0, 1
E_ARG, E_TRUNCATED, E_FRAG, E_RPC, E_AUTH, E_PAD, E_SIZE = -1, -2, -3, -4, -5, -6, -7
E_TRAILING, E_XID, E_PTR, E_CAPACITY, E_PROC = -8, -9, -10, -11, -12

# schema item kinds
K_U32, K_U64, K_OPAQUE_VAR, K_OPAQUE_FIX = 1, 2, 3, 4
N_BUILTIN = 3  # or_builtin_schemas: HtoD, DtoH, HtoD stripe
K_I32_VAR, K_U32_VAR, K_F32_VAR, K_I64_VAR, K_U64_VAR, K_F64_VAR = 5, 6, 7, 8, 9, 10
K_I32_FIX, K_U32_FIX, K_F32_FIX, K_I64_FIX, K_U64_FIX, K_F64_FIX = 11, 12, 13, 14, 15, 16
MAX_ITEMS = 8

ELEM_SIZE = {K_OPAQUE_VAR: 1, K_OPAQUE_FIX: 1, **{k: 4 for k in (5, 6, 7, 11, 12, 13)},
             **{k: 8 for k in (8, 9, 10, 14, 15, 16)}}


def build(force: bool = False) -> str:
    """Compiles oracle.c with gcc into liboracle.so (plain -O1; not tuned)."""
    if force or not os.path.exists(LIBPATH) or os.path.getmtime(LIBPATH) < os.path.getmtime(SRC):
        subprocess.check_call(["gcc", "-O1", "-std=c99", "-Wall", "-shared", "-fPIC", "-o", LIBPATH, SRC])
    return LIBPATH


class Frag(C.Structure):
    _fields_ = [("phys", C.c_uint64), ("lstart", C.c_uint64), ("len", C.c_uint32), ("last", C.c_uint32),
                ("rec", C.c_uint32), ("pad_", C.c_uint32)]


class Rec(C.Structure):
    _fields_ = [("begin", C.c_uint64), ("end", C.c_uint64), ("len", C.c_uint64), ("frag0", C.c_uint32),
                ("nfrags", C.c_uint32)]


class Schema(C.Structure):
    _fields_ = [("proc", C.c_uint32), ("n_items", C.c_uint32), ("items", C.c_uint32 * MAX_ITEMS)]


class Cfg(C.Structure):
    _fields_ = [("prog", C.c_uint32), ("vers", C.c_uint32), ("strict", C.c_int), ("proc_h2d", C.c_uint32),
                ("proc_d2h", C.c_uint32), ("proc_stripe", C.c_uint32)]


class Call(C.Structure):
    _fields_ = [("status", C.c_int32), ("xid", C.c_uint32), ("proc", C.c_uint32), ("n_items", C.c_uint32),
                ("kind", C.c_uint32 * MAX_ITEMS), ("off", C.c_uint64 * MAX_ITEMS),
                ("count", C.c_uint64 * MAX_ITEMS), ("value", C.c_uint64 * MAX_ITEMS), ("end", C.c_uint64)]


class ServeRec(C.Structure):
    _fields_ = [("status", C.c_int32), ("reply_err", C.c_int32), ("ring", C.c_uint32), ("xid", C.c_uint32),
                ("proc", C.c_uint32), ("pad_", C.c_uint32), ("reply_off", C.c_uint64),
                ("reply_wire", C.c_uint64)]


_lib = None
u8p = C.POINTER(C.c_uint8)
u64 = C.c_uint64


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        L.or_be32.restype = C.c_uint32
        L.or_be32.argtypes = [u8p]
        for name in ("or_xdr_put_u32",):
            getattr(L, name).restype = u64
            getattr(L, name).argtypes = [u8p, u64, C.c_uint32]
        L.or_xdr_put_u64.restype = u64
        L.or_xdr_put_u64.argtypes = [u8p, u64, u64]
        L.or_xdr_put_opaque_fix.restype = u64
        L.or_xdr_put_opaque_fix.argtypes = [u8p, u64, u8p, u64]
        L.or_xdr_put_opaque_var.restype = u64
        L.or_xdr_put_opaque_var.argtypes = [u8p, u64, u8p, C.c_uint32]
        L.or_xdr_put_array.restype = u64
        L.or_xdr_put_array.argtypes = [u8p, u64, u8p, C.c_uint32, C.c_uint32, C.c_int]
        L.or_rpc_put_call_header.restype = u64
        L.or_rpc_put_call_header.argtypes = [u8p, u64, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32,
                                             C.c_uint32, u8p, C.c_uint32, C.c_uint32, u8p, C.c_uint32]
        L.or_rpc_put_reply_header.restype = u64
        L.or_rpc_put_reply_header.argtypes = [u8p, u64, C.c_uint32]
        L.or_frame_count.restype = u64
        L.or_frame_count.argtypes = [u64, C.c_uint32]
        L.or_frame_wire_size.restype = u64
        L.or_frame_wire_size.argtypes = [u64, C.c_uint32]
        L.or_frame_record.restype = u64
        L.or_frame_record.argtypes = [u8p, u64, C.c_uint32, u8p]
        L.or_frame_record_lens.restype = u64
        L.or_frame_record_lens.argtypes = [u8p, u64, C.POINTER(C.c_uint32), u64, u8p]
        L.or_frame_scan.restype = C.c_int
        L.or_frame_scan.argtypes = [u8p, u64, u64, u64, u64, C.c_uint32, C.c_uint32, C.POINTER(Frag),
                                    C.POINTER(C.c_uint32), C.POINTER(Rec), C.POINTER(C.c_uint32),
                                    C.POINTER(C.c_uint64)]
        L.or_record_logical.restype = None
        L.or_record_logical.argtypes = [u8p, u64, C.POINTER(Frag), C.POINTER(Rec), u8p]
        L.or_parse_call.restype = C.c_int
        L.or_parse_call.argtypes = [u8p, u64, C.POINTER(Cfg), C.POINTER(Schema), C.c_uint32, C.POINTER(Call)]
        L.or_builtin_schemas.restype = None
        L.or_builtin_schemas.argtypes = [C.POINTER(Cfg), C.POINTER(Schema)]
        L.or_decode_memcpy_h2d.restype = C.c_int
        L.or_decode_memcpy_h2d.argtypes = [u8p, C.POINTER(Call), C.POINTER(Cfg), u8p, u64, C.POINTER(C.c_uint64)]
        L.or_decode_item.restype = C.c_int
        L.or_decode_item.argtypes = [u8p, C.POINTER(Call), C.c_uint32, C.c_uint32, u8p, u64,
                                     C.POINTER(C.c_uint64)]
        L.or_reply_logical_size.restype = u64
        L.or_reply_logical_size.argtypes = [u64, C.c_int32]
        L.or_encode_memcpy_d2h.restype = u64
        L.or_encode_memcpy_d2h.argtypes = [C.c_uint32, u8p, C.c_uint32, C.c_int32, C.c_uint32, u8p]
        L.or_encode_array_reply.restype = u64
        L.or_encode_array_reply.argtypes = [C.c_uint32, u8p, C.c_uint32, C.c_uint32, C.c_int32, C.c_uint32, u8p]
        L.or_encode_reply_item.restype = u64
        L.or_encode_reply_item.argtypes = [C.c_uint32, C.c_int32, C.c_uint32, u64, u8p, C.c_uint32, C.c_uint32, u8p]
        L.or_serve.restype = C.c_int
        L.or_serve.argtypes = [C.c_uint32, C.POINTER(u8p), C.POINTER(C.c_uint64), C.POINTER(C.c_uint64),
                               C.POINTER(C.c_uint64), u64, C.c_uint32, C.c_uint32, C.POINTER(Cfg),
                               C.POINTER(Schema), C.c_uint32, u8p, u64, u64, C.POINTER(u8p),
                               C.POINTER(C.c_uint64), C.POINTER(C.c_uint64), C.c_uint32, C.POINTER(C.c_int32),
                               C.POINTER(C.c_uint64), C.POINTER(C.c_uint64), C.POINTER(ServeRec), C.c_uint32,
                               C.POINTER(C.c_uint32)]
        _lib = L
    return _lib


def _buf(data) -> np.ndarray:
    """Contiguous uint8 view of bytes / bytearray / numpy data."""
    if isinstance(data, np.ndarray):
        return np.ascontiguousarray(data).view(np.uint8).reshape(-1)
    return np.frombuffer(bytes(data), dtype=np.uint8).copy()


def _p(a: np.ndarray):
    return a.ctypes.data_as(u8p)


# ------------------------------------------------------------------ XDR primitives (RFC 4506)

def put_u32(v: int) -> bytes:
    out = np.zeros(4, np.uint8)
    lib().or_xdr_put_u32(_p(out), 0, v & 0xFFFFFFFF)
    return out.tobytes()


def put_u64(v: int) -> bytes:
    out = np.zeros(8, np.uint8)
    lib().or_xdr_put_u64(_p(out), 0, v & 0xFFFFFFFFFFFFFFFF)
    return out.tobytes()


def put_opaque_fix(data) -> bytes:
    d = _buf(data)
    out = np.zeros(len(d) + 4, np.uint8)
    n = lib().or_xdr_put_opaque_fix(_p(out), 0, _p(d), len(d))
    return out[:n].tobytes()


def put_opaque_var(data) -> bytes:
    d = _buf(data)
    out = np.zeros(len(d) + 8, np.uint8)
    n = lib().or_xdr_put_opaque_var(_p(out), 0, _p(d), len(d))
    return out[:n].tobytes()


def put_array(elems: np.ndarray, with_count: bool = True) -> bytes:
    """elems: a numpy array of 4- or 8-byte elements in host order; written big-endian."""
    e = np.ascontiguousarray(elems)
    es = e.dtype.itemsize
    assert es in (4, 8)
    out = np.zeros(len(e) * es + 4, np.uint8)
    n = lib().or_xdr_put_array(_p(out), 0, e.ctypes.data_as(u8p), len(e), es, int(with_count))
    return out[:n].tobytes()


def call_header(xid: int, prog: int, vers: int, proc: int, cred=(0, b""), verf=(0, b"")) -> bytes:
    cb, vb = _buf(cred[1]), _buf(verf[1])
    out = np.zeros(40 + len(cb) + len(vb) + 8, np.uint8)
    n = lib().or_rpc_put_call_header(_p(out), 0, xid, prog, vers, proc, cred[0], _p(cb), len(cb), verf[0],
                                     _p(vb), len(vb))
    return out[:n].tobytes()


def reply_header(xid: int) -> bytes:
    out = np.zeros(24, np.uint8)
    lib().or_rpc_put_reply_header(_p(out), 0, xid)
    return out.tobytes()


def encode_item(kind: int, value) -> bytes:
    """One schema item: U32/U64 take an int, opaque kinds bytes, array kinds a numpy array."""
    if kind == K_U32:
        return put_u32(value)
    if kind == K_U64:
        return put_u64(value)
    if kind == K_OPAQUE_VAR:
        return put_opaque_var(value)
    if kind == K_OPAQUE_FIX:
        return put_opaque_fix(value)
    if K_I32_VAR <= kind <= K_F64_VAR:
        return put_array(value, True)
    return put_array(value, False)


def item_code(kind: int, fixed: int = 0) -> int:
    return kind | (fixed << 8)


# ------------------------------------------------------------------ record marking (RFC 5531 §11)

def frame_count(n: int, F: int) -> int:
    return int(lib().or_frame_count(n, F))


def wire_size(n: int, F: int) -> int:
    return int(lib().or_frame_wire_size(n, F))


def frame(L, F: int) -> bytes:
    d = _buf(L)
    out = np.zeros(wire_size(len(d), F), np.uint8)
    n = lib().or_frame_record(_p(d), len(d), F, _p(out))
    return out[:n].tobytes()


def frame_lens(L, lens) -> bytes:
    d = _buf(L)
    ln = np.ascontiguousarray(np.asarray(lens, dtype=np.uint32))
    assert int(ln.sum()) == len(d) and len(ln) >= 1
    out = np.zeros(len(d) + 4 * len(ln), np.uint8)
    n = lib().or_frame_record_lens(_p(d), len(d), ln.ctypes.data_as(C.POINTER(C.c_uint32)), len(ln), _p(out))
    return out[:n].tobytes()


@dataclass
class ScanResult:
    status: int
    consumed: int
    frags: list  # of dicts phys, lstart, len, last, rec
    recs: list   # of dicts begin, end, len, frag0, nfrags


def frame_scan(ring: np.ndarray, head: int, tail: int, max_record_bytes: int = 1 << 32,
               max_frags: int = 1 << 16, max_records: int = 1 << 14) -> ScanResult:
    r = _buf(ring)
    cap = len(r)
    frags = (Frag * max(1, max_frags))()
    recs = (Rec * max(1, max_records))()
    nf, nr, cons = C.c_uint32(), C.c_uint32(), C.c_uint64()
    st = lib().or_frame_scan(_p(r), cap, head, tail, max_record_bytes, max_frags, max_records, frags,
                             C.byref(nf), recs, C.byref(nr), C.byref(cons))
    fl = [dict(phys=f.phys, lstart=f.lstart, len=f.len, last=f.last, rec=f.rec) for f in frags[: nf.value]]
    rl = [dict(begin=x.begin, end=x.end, len=x.len, frag0=x.frag0, nfrags=x.nfrags) for x in recs[: nr.value]]
    return ScanResult(st, cons.value, fl, rl)


def record_logical(ring: np.ndarray, scan: ScanResult, i: int) -> bytes:
    r = _buf(ring)
    rec = scan.recs[i]
    nf = len(scan.frags)
    frags = (Frag * max(1, nf))()
    for j, f in enumerate(scan.frags):
        frags[j] = Frag(f["phys"], f["lstart"], f["len"], f["last"], f["rec"], 0)
    rr = Rec(rec["begin"], rec["end"], rec["len"], rec["frag0"], rec["nfrags"])
    out = np.zeros(max(1, rec["len"]), np.uint8)
    lib().or_record_logical(_p(r), len(r), frags, C.byref(rr), _p(out))
    return out[: rec["len"]].tobytes()


# ------------------------------------------------------------------ CALL parse + decode

@dataclass
class Config:
    prog: int = 0x20000099
    vers: int = 1
    strict: bool = True
    proc_h2d: int = 1
    proc_d2h: int = 2
    proc_stripe: int = 3  # the HtoD stripe (NEXT-1, reading R22); 0 disables it
    frag_payload: int = 65536
    user_schemas: dict = field(default_factory=dict)  # proc -> list of item codes

    def c(self) -> Cfg:
        return Cfg(self.prog, self.vers, int(self.strict), self.proc_h2d, self.proc_d2h, self.proc_stripe)

    def schemas(self):
        n = N_BUILTIN + len(self.user_schemas)
        arr = (Schema * n)()
        cfg = self.c()
        lib().or_builtin_schemas(C.byref(cfg), arr)
        for i, (proc, items) in enumerate(self.user_schemas.items()):
            assert len(items) <= MAX_ITEMS
            arr[N_BUILTIN + i].proc = proc
            arr[N_BUILTIN + i].n_items = len(items)
            for j, it in enumerate(items):
                arr[N_BUILTIN + i].items[j] = it
        return arr, n


def parse_call(L: bytes, cfg: Config) -> Call:
    d = _buf(L)
    arr, n = cfg.schemas()
    c = Call()
    cc = cfg.c()
    lib().or_parse_call(_p(d) if len(d) else _p(np.zeros(1, np.uint8)), len(d), C.byref(cc), arr, n, C.byref(c))
    return c


def decode_memcpy_h2d(L: bytes, call: Call, cfg: Config, dst_bytes: int):
    d = _buf(L) if len(L) else np.zeros(1, np.uint8)
    out = np.zeros(max(1, dst_bytes), np.uint8)
    copied = C.c_uint64()
    cc = cfg.c()
    st = lib().or_decode_memcpy_h2d(_p(d), C.byref(call), C.byref(cc), _p(out), dst_bytes, C.byref(copied))
    return st, out[: copied.value].tobytes()


def decode_item(L: bytes, call: Call, arg_no: int, kind: int, max_count: int):
    """Returns (status, uint8 array in host byte order of count*elem_size bytes)."""
    d = _buf(L) if len(L) else np.zeros(1, np.uint8)
    es = ELEM_SIZE.get(kind, 1)
    out = np.zeros(max(1, min(max_count, call.count[arg_no] if arg_no < MAX_ITEMS else 0) * es), np.uint8)
    cnt = C.c_uint64()
    st = lib().or_decode_item(_p(d), C.byref(call), arg_no, kind, _p(out), max_count, C.byref(cnt))
    return st, out[: cnt.value * es]


# ------------------------------------------------------------------ encode

def encode_memcpy_d2h(xid: int, src, err: int, F: int) -> bytes:
    s = _buf(src) if src is not None else np.zeros(0, np.uint8)
    n = len(s) if err == 0 else 0
    sp = _p(s) if len(s) else _p(np.zeros(1, np.uint8))
    w = lib().or_encode_memcpy_d2h(xid, sp, n, err, F, None)
    out = np.zeros(w, np.uint8)
    lib().or_encode_memcpy_d2h(xid, sp, n, err, F, _p(out))
    return out.tobytes()


def encode_array_reply(xid: int, elems: np.ndarray, err: int, F: int) -> bytes:
    e = np.ascontiguousarray(elems)
    es = e.dtype.itemsize
    ep = e.ctypes.data_as(u8p) if len(e) else _p(np.zeros(8, np.uint8))
    w = lib().or_encode_array_reply(xid, ep, len(e), es, err, F, None)
    out = np.zeros(w, np.uint8)
    lib().or_encode_array_reply(xid, ep, len(e), es, err, F, _p(out))
    return out.tobytes()


def encode_reply_item(xid: int, err: int, kind: int, value=0, elems=None, F: int = 65536) -> bytes:
    """Generic REPLY with one result item (see or_encode_reply_item)."""
    if elems is None:
        e, count = np.zeros(8, np.uint8), 0
    else:
        e = np.ascontiguousarray(elems)
        count = len(e)
        e = e.view(np.uint8) if e.size else np.zeros(8, np.uint8)
    w = lib().or_encode_reply_item(xid, err, kind, value & 0xFFFFFFFFFFFFFFFF, _p(e), count, F, None)
    out = np.zeros(w, np.uint8)
    lib().or_encode_reply_item(xid, err, kind, value & 0xFFFFFFFFFFFFFFFF, _p(e), count, F, _p(out))
    return out.tobytes()


def encode_call(xid: int, proc: int, items, cfg: Config, F: int | None = None, lens=None,
                cred=(0, b""), verf=(0, b"")) -> bytes:
    """Builds the logical CALL (header + items as (kind, value) pairs) and frames it."""
    L = call_header(xid, cfg.prog, cfg.vers, proc, cred, verf) + b"".join(encode_item(k, v) for k, v in items)
    if lens is not None:
        return frame_lens(L, lens)
    return frame(L, F if F is not None else cfg.frag_payload)


# ------------------------------------------------------------------ server step

def serve(rings, cfg: Config, region: np.ndarray, region_base: int, send_caps, out_off, *,
          max_record_bytes: int = 1 << 32, max_frags_per_ring: int = 1 << 16,
          max_records_per_ring: int = 1 << 14, with_send_rings: bool = True):
    """rings: list of (uint8 ring array (len = cap, power of two), head, tail).
    Mutates `region` (uint8 array standing for device memory at address region_base).
    Returns dict with scan_status, consumed, reply_bytes, records (list of dicts), send (list of arrays)."""
    n = len(rings)
    rbufs = [_buf(r[0]) for r in rings]
    ring_ptrs = (u8p * n)(*[_p(b) for b in rbufs])
    caps = (C.c_uint64 * n)(*[len(b) for b in rbufs])
    heads = (C.c_uint64 * n)(*[r[1] for r in rings])
    tails = (C.c_uint64 * n)(*[r[2] for r in rings])
    sends = [np.zeros(int(c), np.uint8) for c in send_caps]
    send_ptrs = (u8p * n)(*[_p(s) for s in sends]) if with_send_rings else None
    scaps = (C.c_uint64 * n)(*send_caps)
    offs = (C.c_uint64 * n)(*out_off)
    sst = (C.c_int32 * n)()
    cons = (C.c_uint64 * n)()
    rbytes = (C.c_uint64 * n)()
    max_out = max_records_per_ring * n
    recs = (ServeRec * max(1, max_out))()
    nout = C.c_uint32()
    arr, ns = cfg.schemas()
    cc = cfg.c()
    assert region.dtype == np.uint8 and region.flags.c_contiguous
    lib().or_serve(n, ring_ptrs, caps, heads, tails, max_record_bytes, max_frags_per_ring, max_records_per_ring,
                   C.byref(cc), C.cast(C.byref(arr, N_BUILTIN * C.sizeof(Schema)), C.POINTER(Schema)), ns - N_BUILTIN,
                   _p(region) if region.size else _p(np.zeros(1, np.uint8)), region_base, region.size,
                   send_ptrs, scaps, offs, cfg.frag_payload, sst, cons, rbytes, recs, max_out, C.byref(nout))
    out = [dict(status=r.status, reply_err=r.reply_err, ring=r.ring, xid=r.xid, proc=r.proc,
                reply_off=r.reply_off, reply_wire=r.reply_wire) for r in recs[: nout.value]]
    return dict(scan_status=list(sst), consumed=list(cons), reply_bytes=list(rbytes), records=out, send=sends)
