"""Python binding of the crk C ABI (include/crk.h): argument marshalling only.

Every step of the data path runs in libcrk.so's sm_100a kernels; this module converts torch tensors
(device memory, pinned host memory, streams) into the plain pointers and sizes the C ABI takes.  There
is no CPU fallback: if libcrk.so is missing, importing a function that needs it raises.
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass

import numpy as np
import torch

PKG = os.path.dirname(os.path.abspath(__file__))
LIBPATH = os.environ.get("CRK_LIB") or os.path.join(PKG, "lib", "libcrk.so")  # CRK_LIB: a diagnostic / A-B build variant

OK, INCOMPLETE = 0, 1
E_ARG, E_TRUNCATED, E_FRAG, E_RPC, E_AUTH, E_PAD, E_SIZE = -1, -2, -3, -4, -5, -6, -7
E_TRAILING, E_XID, E_PTR, E_CAPACITY, E_PROC, E_CUDA = -8, -9, -10, -11, -12, -100

K_U32, K_U64, K_OPAQUE_VAR, K_OPAQUE_FIX = 1, 2, 3, 4
K_I32_VAR, K_U32_VAR, K_F32_VAR, K_I64_VAR, K_U64_VAR, K_F64_VAR = 5, 6, 7, 8, 9, 10
K_I32_FIX, K_U32_FIX, K_F32_FIX, K_I64_FIX, K_U64_FIX, K_F64_FIX = 11, 12, 13, 14, 15, 16
MAX_ITEMS, MAX_RINGS = 8, 64
ELEM_SIZE = {K_OPAQUE_VAR: 1, K_OPAQUE_FIX: 1, **{k: 4 for k in (5, 6, 7, 11, 12, 13)},
             **{k: 8 for k in (8, 9, 10, 14, 15, 16)}}
TYPED = {"i32": (K_I32_VAR, torch.int32), "u32": (K_U32_VAR, torch.uint32), "i64": (K_I64_VAR, torch.int64),
         "u64": (K_U64_VAR, torch.uint64), "f32": (K_F32_VAR, torch.float32), "f64": (K_F64_VAR, torch.float64)}


class CrkError(RuntimeError):
    def __init__(self, status: int, what: str = ""):
        self.status = status
        msg = f"{what}: crk status {status} ({strerror(status)})"
        if status == E_CUDA:
            msg += f", cudaError {lib().crk_last_cuda_error()}"
        super().__init__(msg)


class Config(C.Structure):
    _fields_ = [("frag_payload", C.c_uint32), ("strict", C.c_int32), ("max_record_bytes", C.c_uint64),
                ("prog", C.c_uint32), ("vers", C.c_uint32), ("proc_h2d", C.c_uint32), ("proc_d2h", C.c_uint32),
                ("scan_stride_guess", C.c_uint32), ("tile_bytes", C.c_uint32), ("max_jobs", C.c_uint32),
                ("ctas_per_sm", C.c_uint32), ("scan_threads", C.c_uint32), ("mover_stages", C.c_uint32),
                ("mover_run", C.c_uint32), ("mover_tail_tiles", C.c_uint32), ("mover_reserve_ctas", C.c_uint32),
                ("fused_front_max_records", C.c_uint32), ("scan_chunking", C.c_uint32), ("fused_front_max_window", C.c_uint64),
                ("proc_h2d_stripe", C.c_uint32), ("mover_max_ctas", C.c_uint32),
                ("fused_front_max_frags", C.c_uint32), ("lean_steps", C.c_uint32), ("lean_backoff", C.c_uint32)]


class CRing(C.Structure):
    _fields_ = [("base", C.c_void_p), ("cap", C.c_uint64)]


class RingResult(C.Structure):
    _fields_ = [("status", C.c_int32), ("n_records", C.c_uint32), ("n_frags", C.c_uint32), ("rec_base", C.c_uint32),
                ("consumed", C.c_uint64), ("reply_bytes", C.c_uint64)]


class IndexView(C.Structure):
    _fields_ = [("max_rings", C.c_uint32), ("frags_per_ring", C.c_uint32), ("recs_per_ring", C.c_uint32),
                ("max_records", C.c_uint32)] + [(n, C.c_void_p) for n in (
                    "frag_phys", "frag_lstart", "frag_hdr", "rec_begin", "rec_len", "rec_frag0", "rec_nfrags",
                    "p_slot", "p_ring", "p_xid", "p_proc", "p_status", "p_nitems", "p_kind", "p_off", "p_count",
                    "p_value", "serve_status", "serve_reply_err", "serve_reply_off", "serve_reply_wire",
                    "ring_results", "total_records")]


class ItemReq(C.Structure):
    _fields_ = [("xid", C.c_uint32), ("arg_no", C.c_uint32), ("kind", C.c_uint32), ("pad_", C.c_uint32),
                ("dst", C.c_void_p), ("max_count", C.c_uint64), ("count", C.c_void_p), ("status", C.c_void_p)]


class ItemSrc(C.Structure):
    _fields_ = [("kind", C.c_uint32), ("pad_", C.c_uint32), ("value", C.c_uint64), ("src", C.c_void_p),
                ("count", C.c_uint64)]


class ReplyReq(C.Structure):
    _fields_ = [("xid", C.c_uint32), ("err", C.c_int32), ("kind", C.c_uint32), ("pad_", C.c_uint32),
                ("value", C.c_uint64), ("src", C.c_void_p), ("count", C.c_uint64)]


class ServerBell(C.Structure):
    """crk_server_bell (include/crk.h): the persistent server's doorbell and result block."""
    _fields_ = [("seq", C.c_uint64), ("stop", C.c_uint64), ("head", C.c_uint64 * MAX_RINGS),
                ("tail", C.c_uint64 * MAX_RINGS), ("send_off", C.c_uint64 * MAX_RINGS), ("done_seq", C.c_uint64),
                ("status", C.c_int32), ("pad_", C.c_uint32), ("t_begin_ns", C.c_uint64), ("t_end_ns", C.c_uint64),
                ("t_phase_ns", C.c_uint64 * 5), ("res", RingResult * MAX_RINGS)]


_lib = None
vp, u32, u64, i32 = C.c_void_p, C.c_uint32, C.c_uint64, C.c_int32


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIBPATH):
            raise RuntimeError(f"crk CUDA extension missing ({LIBPATH}); run __graft_entry__.build()")
        L = C.CDLL(LIBPATH)
        sig = {
            "crk_config_init": (None, [C.POINTER(Config)]),
            "crk_ctx_create": (C.c_int, [C.c_int, C.POINTER(Config), C.POINTER(vp)]),
            "crk_ctx_destroy": (None, [vp]),
            "crk_proc_schema_register": (C.c_int, [vp, u32, C.POINTER(u32), u32]),
            "crk_index_create": (C.c_int, [vp, u32, u32, u32, C.POINTER(vp)]),
            "crk_index_destroy": (None, [vp]),
            "crk_index_get_view": (C.c_int, [vp, C.POINTER(IndexView)]),
            "crk_index_ring_results": (C.c_int, [vp, u32, C.POINTER(RingResult), vp]),
            "crk_index_ring_results_async": (C.c_int, [vp, u32, vp, vp]),
            "crk_ring_copy": (C.c_int, [CRing, CRing, u64, u64, vp]),
            "crk_rpc_frame_scan": (C.c_int, [vp, vp, u32, C.POINTER(CRing), C.POINTER(u64), C.POINTER(u64), vp]),
            "crk_xdr_decode_memcpy_h2d": (C.c_int, [vp, vp, u32, vp, u64, vp, vp, vp]),
            "crk_xdr_decode_memcpy_h2d_batch": (C.c_int, [vp, vp, u32, vp, vp, vp, vp, vp, vp]),
            "crk_xdr_decode_opaque": (C.c_int, [vp, vp, u32, u32, vp, u64, vp, vp, vp]),
            "crk_xdr_decode_items_batch": (C.c_int, [vp, vp, u32, vp, vp]),
            "crk_wire_size_d2h": (u64, [u64, i32, u32]),
            "crk_xdr_encode_memcpy_d2h": (C.c_int, [vp, u32, vp, u64, i32, CRing, u64, C.POINTER(u64), vp]),
            "crk_xdr_encode_memcpy_d2h_batch": (C.c_int, [vp, u32, vp, vp, vp, vp, CRing, u64, vp, vp, vp]),
            "crk_rpc_encode_replies_batch": (C.c_int, [vp, u32, vp, CRing, u64, vp, vp, vp]),
            "crk_rpc_encode_call": (C.c_int, [vp, u32, u32, C.POINTER(ItemSrc), u32, C.POINTER(u32), u32, CRing, u64,
                                              C.POINTER(u64), vp]),
            "crk_call_logical_size": (u64, [C.POINTER(ItemSrc), u32]),
            "crk_serve": (C.c_int, [vp, vp, u32, C.POINTER(CRing), C.POINTER(u64), C.POINTER(u64), C.POINTER(CRing),
                                    C.POINTER(u64), u64, u64, vp]),
            "crk_serve_graph_create": (C.c_int, [vp, vp, u32, C.POINTER(CRing), C.POINTER(CRing), u64, u64, vp,
                                                 C.POINTER(vp)]),
            "crk_graph_launch": (C.c_int, [vp, vp]),
            "crk_server_start": (C.c_int, [vp, vp, u32, C.POINTER(CRing), C.POINTER(CRing), u64, u64, vp, vp,
                                           C.POINTER(vp)]),
            "crk_server_stop": (C.c_int, [vp]),
            "crk_server_step": (C.c_int, [vp, C.POINTER(u64), C.POINTER(u64), C.POINTER(u64), u64]),
            "crk_graph_destroy": (None, [vp]),
            "crk_host_alloc": (C.c_int, [u64, C.POINTER(vp)]),
            "crk_host_free": (None, [vp]),
            "crk_copy_to_host": (C.c_int, [vp, vp, u64]),
            "crk_strerror": (C.c_char_p, [C.c_int]),
            "crk_last_cuda_error": (C.c_int, []),
            "crk_kernel_launches": (C.c_int, []),
            "crk_profile_enable": (C.c_int, [C.c_int]),
            "crk_profile_read": (C.c_int, [C.POINTER(C.c_double), C.POINTER(u32)]),
            "crk_version": (C.c_char_p, []),
            "crk_debug_counters": (C.c_int, [vp, C.POINTER(u32)]),  # diagnostic, not in include/crk.h
            "crk_debug_index_stats": (C.c_int, [vp, C.POINTER(u32)]),  # diagnostic, not in include/crk.h
            "crk_debug_index_ms": (C.c_int, [vp, C.POINTER(vp), C.POINTER(u32)]),  # diagnostic
        }
        for t in ("i32", "u32", "i64", "u64", "f32", "f64"):
            sig[f"crk_xdr_decode_array_{t}"] = (C.c_int, [vp, vp, u32, u32, vp, u64, vp, vp, vp])
            sig[f"crk_xdr_encode_array_{t}"] = (C.c_int, [vp, u32, vp, u64, i32, CRing, u64, C.POINTER(u64), vp])
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def strerror(status: int) -> str:
    return lib().crk_strerror(status).decode()


def kernel_launches() -> int:
    return int(lib().crk_kernel_launches())


PROF_STAGES = ("scan", "parse", "plan", "move")


def profile_enable(on: bool = True):
    _check(lib().crk_profile_enable(int(on)), "crk_profile_enable")


def profile_read() -> dict:
    """{stage: (device ms summed over timed launches, launches)} since the last read."""
    ms = (C.c_double * 4)()
    n = (u32 * 4)()
    _check(lib().crk_profile_read(ms, n), "crk_profile_read")
    return {s: (ms[i], n[i]) for i, s in enumerate(PROF_STAGES)}


def _check(st: int, what: str):
    if st != OK:
        raise CrkError(st, what)


def _stream(stream) -> int:
    if stream is None:
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, torch.cuda.Stream):
        return stream.cuda_stream
    return int(stream)


def _ptr(t) -> int | None:
    if t is None:
        return None
    if isinstance(t, int):
        return t
    return t.data_ptr()


# ------------------------------------------------------------------ host memory and rings

class HostBuffer:
    """Pinned, mapped host memory (crk_host_alloc); `.np` is a writable numpy view, `.ptr` works in kernels."""

    def __init__(self, nbytes: int):
        p = vp()
        _check(lib().crk_host_alloc(nbytes, C.byref(p)), "crk_host_alloc")
        self.ptr = p.value
        self.nbytes = nbytes
        self.np = np.ctypeslib.as_array(C.cast(p, C.POINTER(C.c_uint8)), shape=(nbytes,))

    def free(self):
        if self.ptr:
            lib().crk_host_free(self.ptr)
            self.ptr = 0

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


class _HostView:
    """Part of a HostBuffer (keeps the buffer alive); `.np` views the part."""

    def __init__(self, buf, np_view):
        self.buf, self.np = buf, np_view


@dataclass
class Ring:
    """A ring: `cap` (power of two >= 256) bytes of device memory or pinned mapped host memory."""
    base: int
    cap: int
    owner: object = None  # keeps the tensor / HostBuffer alive

    @staticmethod
    def device(cap: int, device=None) -> "Ring":
        t = torch.empty(cap, dtype=torch.uint8, device=device or "cuda")
        return Ring(t.data_ptr(), cap, t)

    @staticmethod
    def host(cap: int) -> "Ring":
        h = HostBuffer(cap)
        return Ring(h.ptr, cap, h)

    @staticmethod
    def of(t: torch.Tensor) -> "Ring":
        return Ring(t.data_ptr(), t.numel() * t.element_size(), t)

    def c(self) -> CRing:
        return CRing(self.base, self.cap)

    def sub(self, offset: int, cap: int) -> "Ring":
        """A ring over bytes [offset, offset + cap) of this one's memory (offset 256-aligned, cap a power of two)."""
        assert offset % 256 == 0 and offset + cap <= self.cap and cap & (cap - 1) == 0
        if isinstance(self.owner, torch.Tensor):
            return Ring(self.base + offset, cap, self.owner[offset:offset + cap])
        view = _HostView(self.owner, self.host_view()[offset:offset + cap])
        return Ring(self.base + offset, cap, view)

    def tensor(self) -> torch.Tensor | None:
        return self.owner if isinstance(self.owner, torch.Tensor) else None

    def host_view(self) -> np.ndarray | None:
        return self.owner.np if isinstance(self.owner, (HostBuffer, _HostView)) else None

    def read(self, cursor: int, n: int) -> bytes:
        """Bytes [cursor, cursor + n) with wrap (host-side inspection, for tests)."""
        out = bytearray()
        while n > 0:
            o = cursor % self.cap
            k = min(n, self.cap - o)
            hv = self.host_view()
            if hv is not None:
                out += hv[o:o + k].tobytes()
            else:
                out += self.owner[o:o + k].cpu().numpy().tobytes()
            cursor += k
            n -= k
        return bytes(out)

    def write(self, cursor: int, data: bytes):
        """Host-side fill with wrap (tests/bench setup)."""
        data = np.frombuffer(bytes(data), np.uint8)
        i = 0
        while i < len(data):
            o = (cursor + i) % self.cap
            k = min(len(data) - i, self.cap - o)
            hv = self.host_view()
            if hv is not None:
                hv[o:o + k] = data[i:i + k]
            else:
                self.owner[o:o + k].copy_(torch.from_numpy(data[i:i + k].copy()))
            i += k


def ring_copy(dst: Ring, src: Ring, head: int, tail: int, stream=None):
    """Copy-engine copy of the cursor window [head, tail) from ring src to ring dst (crk_ring_copy)."""
    _check(lib().crk_ring_copy(dst.c(), src.c(), head, tail, _stream(stream)), "crk_ring_copy")


class PinnedResults:
    """Pinned host slots for crk_index_ring_results_async."""

    def __init__(self, n: int):
        self.buf = HostBuffer(C.sizeof(RingResult) * max(1, n))
        self.n = n

    def rows(self) -> list[dict]:
        arr = (RingResult * self.n).from_address(self.buf.ptr)
        return [dict(status=r.status, n_records=r.n_records, n_frags=r.n_frags, rec_base=r.rec_base,
                     consumed=r.consumed, reply_bytes=r.reply_bytes) for r in arr]


def copy_to_host(dev_ptr: int, nbytes: int) -> np.ndarray:
    out = np.empty(max(1, nbytes), np.uint8)
    if nbytes:
        _check(lib().crk_copy_to_host(out.ctypes.data, dev_ptr, nbytes), "crk_copy_to_host")
    return out[:nbytes]


def config(**kw) -> Config:
    c = Config()
    lib().crk_config_init(C.byref(c))
    names = {f for f, _ in Config._fields_}
    for k, v in kw.items():
        if k not in names:  # a ctypes Structure would silently keep a misspelt field as a Python attribute
            raise KeyError(f"crk_config has no field {k!r}")
        setattr(c, k, v)
    return c


def wire_size_d2h(nbytes: int, err: int = 0, frag_payload: int = 65536) -> int:
    return int(lib().crk_wire_size_d2h(nbytes, err, frag_payload))


# ------------------------------------------------------------------ context

class Context:
    def __init__(self, device: int = 0, **cfg):
        self.cfg = config(**cfg)
        h = vp()
        _check(lib().crk_ctx_create(device, C.byref(self.cfg), C.byref(h)), "crk_ctx_create")
        self.h = h.value
        self.device = device

    def close(self):
        if self.h:
            lib().crk_ctx_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def debug_counters(self) -> list[int]:
        """Diagnostic: the context's 16 scratch counters (synchronises the device)."""
        out = (C.c_uint32 * 16)()
        _check(lib().crk_debug_counters(self.h, out), "crk_debug_counters")
        return list(out)

    def register_schema(self, proc: int, items):
        arr = (u32 * max(1, len(items)))(*items)
        _check(lib().crk_proc_schema_register(self.h, proc, arr, len(items)), "crk_proc_schema_register")

    def index(self, max_rings: int = 1, max_frags: int = 1 << 16, max_records: int = 1 << 12) -> "Index":
        return Index(self, max_rings, max_frags, max_records)

    # ---- encode
    @staticmethod
    def _items(items):
        arr = (ItemSrc * max(1, len(items)))()
        keep = []
        for i, (kind, v) in enumerate(items):
            k = kind & 0xFF
            arr[i].kind = kind
            if k in (K_U32, K_U64):
                arr[i].value = int(v) & 0xFFFFFFFFFFFFFFFF
            else:
                t = v
                keep.append(t)
                arr[i].src = t.data_ptr() if t.numel() else None
                arr[i].count = t.numel() if k in (K_OPAQUE_VAR, K_OPAQUE_FIX) and t.element_size() == 1 else (
                    t.numel() * t.element_size() // ELEM_SIZE[k])
        return arr, keep

    def call_logical_size(self, items) -> int:
        arr, _ = self._items(items)
        return int(lib().crk_call_logical_size(arr, len(items)))

    def encode_call(self, xid: int, proc: int, items, out: Ring, out_off: int, frag_lens=None, stream=None) -> int:
        """items: list of (kind, int | device tensor); returns the wire size."""
        arr, keep = self._items(items)
        w = u64()
        lens = None
        nl = 0
        if frag_lens is not None:
            nl = len(frag_lens)
            lens = (u32 * nl)(*[int(x) for x in frag_lens])
        _check(lib().crk_rpc_encode_call(self.h, xid, proc, arr, len(items), lens, nl, out.c(), out_off, C.byref(w),
                                         _stream(stream)), "crk_rpc_encode_call")
        return w.value

    def encode_memcpy_d2h(self, xid: int, src: torch.Tensor | None, err: int, out: Ring, out_off: int,
                          nbytes: int | None = None, stream=None) -> int:
        w = u64()
        n = nbytes if nbytes is not None else (src.numel() * src.element_size() if src is not None else 0)
        _check(lib().crk_xdr_encode_memcpy_d2h(self.h, xid, _ptr(src), n, err, out.c(), out_off, C.byref(w),
                                               _stream(stream)), "crk_xdr_encode_memcpy_d2h")
        return w.value

    def encode_array(self, t: str, xid: int, src: torch.Tensor, err: int, out: Ring, out_off: int, stream=None) -> int:
        w = u64()
        f = getattr(lib(), f"crk_xdr_encode_array_{t}")
        _check(f(self.h, xid, _ptr(src), src.numel(), err, out.c(), out_off, C.byref(w), _stream(stream)),
               f"crk_xdr_encode_array_{t}")
        return w.value

    def encode_memcpy_d2h_batch(self, xids: torch.Tensor, srcs: torch.Tensor, nbytes: torch.Tensor,
                                errs: torch.Tensor | None, out: Ring, out_off: int, wire_offs: torch.Tensor | None,
                                total: torch.Tensor | None, stream=None):
        _check(lib().crk_xdr_encode_memcpy_d2h_batch(self.h, xids.numel(), _ptr(xids), _ptr(srcs), _ptr(nbytes),
                                                     _ptr(errs), out.c(), out_off, _ptr(wire_offs), _ptr(total),
                                                     _stream(stream)), "crk_xdr_encode_memcpy_d2h_batch")

    def encode_replies_batch(self, reqs, out: Ring, out_off: int, wire_offs: torch.Tensor | None = None,
                             total: torch.Tensor | None = None, stream=None) -> torch.Tensor:
        """reqs: list of (xid, err, kind, value, src tensor | None, count).  Marshals them into a device
        crk_reply_req array (kept alive until the stream is synchronised by the caller) and encodes."""
        n = len(reqs)
        arr = (ReplyReq * max(1, n))()
        for i, (xid, err, kind, value, src, count) in enumerate(reqs):
            arr[i] = ReplyReq(xid, err, kind, 0, value & 0xFFFFFFFFFFFFFFFF, _ptr(src), count)
        host = torch.frombuffer(bytearray(arr), dtype=torch.uint8)
        dev = host.to(f"cuda:{self.device}")
        _check(lib().crk_rpc_encode_replies_batch(self.h, n, _ptr(dev), out.c(), out_off, _ptr(wire_offs),
                                                  _ptr(total), _stream(stream)), "crk_rpc_encode_replies_batch")
        return dev


# ------------------------------------------------------------------ index

def _ring_args(rings):
    n = len(rings)
    cr = (CRing * n)(*[r[0].c() for r in rings])
    heads = (u64 * n)(*[int(r[1]) for r in rings])
    tails = (u64 * n)(*[int(r[2]) for r in rings])
    return n, cr, heads, tails


class Index:
    def __init__(self, ctx: Context, max_rings: int, max_frags: int, max_records: int):
        self.ctx = ctx
        h = vp()
        _check(lib().crk_index_create(ctx.h, max_rings, max_frags, max_records, C.byref(h)), "crk_index_create")
        self.h = h.value
        self.max_rings = max_rings
        v = IndexView()
        _check(lib().crk_index_get_view(self.h, C.byref(v)), "crk_index_get_view")
        self.v = v
        self.n_rings = 0

    def close(self):
        if self.h:
            lib().crk_index_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def frame_scan(self, rings, stream=None):
        """rings: list of (Ring, head, tail)."""
        n, cr, heads, tails = _ring_args(rings)
        _check(lib().crk_rpc_frame_scan(self.ctx.h, self.h, n, cr, heads, tails, _stream(stream)),
               "crk_rpc_frame_scan")
        self.n_rings = n

    def serve(self, rings, send_rings, send_offs, region_base: int, region_bytes: int, stream=None):
        n, cr, heads, tails = _ring_args(rings)
        sr = (CRing * n)(*[s.c() for s in send_rings])
        so = (u64 * n)(*[int(o) for o in send_offs])
        _check(lib().crk_serve(self.ctx.h, self.h, n, cr, heads, tails, sr, so, region_base, region_bytes,
                               _stream(stream)), "crk_serve")
        self.n_rings = n

    def serve_graph(self, rings, send_rings, region_base: int, region_bytes: int, doorbell) -> "ServeGraph":
        """Captures one server step reading its cursors from `doorbell` (a device uint64 tensor or a
        HostBuffer of 3 * n_rings uint64: heads | tails | send offsets)."""
        return ServeGraph(self, rings, send_rings, region_base, region_bytes, doorbell)

    def scan_stats(self) -> dict:
        """Diagnostic: rings this index's scans resolved with the chunked multi-CTA scan, and rings that fell
        back to the one-CTA scan (totals since creation; synchronises the device)."""
        out = (C.c_uint32 * 4)()
        _check(lib().crk_debug_index_stats(self.h, out), "crk_debug_index_stats")
        return {"chunked": out[0], "fallback": out[1]}

    def ring_results(self, n: int | None = None, stream=None) -> list[dict]:
        n = self.n_rings if n is None else n
        out = (RingResult * max(1, n))()
        _check(lib().crk_index_ring_results(self.h, n, out, _stream(stream)), "crk_index_ring_results")
        return [dict(status=r.status, n_records=r.n_records, n_frags=r.n_frags, rec_base=r.rec_base,
                     consumed=r.consumed, reply_bytes=r.reply_bytes) for r in out[:n]]

    def ring_results_async(self, out: "PinnedResults", stream=None):
        _check(lib().crk_index_ring_results_async(self.h, out.n, out.buf.ptr, _stream(stream)),
               "crk_index_ring_results_async")

    def tables(self, n_rings: int | None = None, sync: bool = True) -> dict:
        """Host copies of the index tables after synchronising the device (tests / inspection).  sync=False
        skips the device-wide synchronisation (a persistent server owning the index is still running; its
        tables are complete once its doorbell shows the step done)."""
        if sync:
            torch.cuda.synchronize()
        n_rings = self.n_rings if n_rings is None else n_rings
        v = self.v
        res = self.ring_results(n_rings)
        total = int(copy_to_host(v.total_records, 4).view(np.uint32)[0])
        frags, recs = [], []
        for r, rr in enumerate(res):
            fb, rb = r * v.frags_per_ring, r * v.recs_per_ring
            nf, nr = rr["n_frags"], rr["n_records"]
            g = lambda p, dt, base, cnt: copy_to_host(p + base * np.dtype(dt).itemsize,
                                                      cnt * np.dtype(dt).itemsize).view(dt)
            frags.append(dict(phys=g(v.frag_phys, np.uint64, fb, nf), lstart=g(v.frag_lstart, np.uint64, fb, nf),
                              hdr=g(v.frag_hdr, np.uint32, fb, nf)))
            recs.append(dict(begin=g(v.rec_begin, np.uint64, rb, nr), len=g(v.rec_len, np.uint64, rb, nr),
                             frag0=g(v.rec_frag0, np.uint32, rb, nr) - fb, nfrags=g(v.rec_nfrags, np.uint32, rb, nr)))
        d = lambda p, dt, w=1: copy_to_host(p, total * w * np.dtype(dt).itemsize).view(dt).reshape(total, w) if w > 1 \
            else copy_to_host(p, total * np.dtype(dt).itemsize).view(dt)
        parsed = dict(slot=d(v.p_slot, np.uint32), ring=d(v.p_ring, np.uint32), xid=d(v.p_xid, np.uint32),
                      proc=d(v.p_proc, np.uint32), status=d(v.p_status, np.int32), nitems=d(v.p_nitems, np.uint32),
                      kind=d(v.p_kind, np.uint32, MAX_ITEMS), off=d(v.p_off, np.uint64, MAX_ITEMS),
                      count=d(v.p_count, np.uint64, MAX_ITEMS), value=d(v.p_value, np.uint64, MAX_ITEMS),
                      serve_status=d(v.serve_status, np.int32), serve_reply_err=d(v.serve_reply_err, np.int32),
                      serve_reply_off=d(v.serve_reply_off, np.uint64),
                      serve_reply_wire=d(v.serve_reply_wire, np.uint64))
        return dict(rings=res, total=total, frags=frags, recs=recs, parsed=parsed)

    # ---- decode
    def decode_memcpy_h2d(self, xid: int, dst: torch.Tensor | int | None, dst_bytes: int, status: torch.Tensor,
                          copied: torch.Tensor | None = None, stream=None):
        _check(lib().crk_xdr_decode_memcpy_h2d(self.ctx.h, self.h, xid, _ptr(dst), dst_bytes, _ptr(status),
                                               _ptr(copied), _stream(stream)), "crk_xdr_decode_memcpy_h2d")

    def decode_memcpy_h2d_batch(self, xids: torch.Tensor, dsts: torch.Tensor, dst_bytes: torch.Tensor,
                                statuses: torch.Tensor, copied: torch.Tensor | None = None, stream=None):
        _check(lib().crk_xdr_decode_memcpy_h2d_batch(self.ctx.h, self.h, xids.numel(), _ptr(xids), _ptr(dsts),
                                                     _ptr(dst_bytes), _ptr(statuses), _ptr(copied), _stream(stream)),
               "crk_xdr_decode_memcpy_h2d_batch")

    def decode_array(self, t: str, xid: int, arg_no: int, dst: torch.Tensor | None, max_count: int,
                     count: torch.Tensor | None, status: torch.Tensor, stream=None):
        f = getattr(lib(), f"crk_xdr_decode_array_{t}")
        _check(f(self.ctx.h, self.h, xid, arg_no, _ptr(dst), max_count, _ptr(count), _ptr(status), _stream(stream)),
               f"crk_xdr_decode_array_{t}")

    def decode_opaque(self, xid: int, arg_no: int, dst: torch.Tensor | None, max_count: int,
                      count: torch.Tensor | None, status: torch.Tensor, stream=None):
        _check(lib().crk_xdr_decode_opaque(self.ctx.h, self.h, xid, arg_no, _ptr(dst), max_count, _ptr(count),
                                           _ptr(status), _stream(stream)), "crk_xdr_decode_opaque")

    def decode_items_batch(self, reqs: list[tuple], stream=None) -> torch.Tensor:
        """reqs: list of (xid, arg_no, kind, dst ptr, max_count, count ptr|None, status ptr).  The request
        array is staged to the device; returns that device buffer (keep it alive until the stream syncs)."""
        n = len(reqs)
        arr = (ItemReq * max(1, n))()
        for i, (xid, arg, kind, dst, mc, cnt, st) in enumerate(reqs):
            arr[i] = ItemReq(xid, arg, kind, 0, dst, mc, cnt, st)
        host = torch.frombuffer(bytearray(arr), dtype=torch.uint8)
        dev = host.to(f"cuda:{self.ctx.device}", non_blocking=False)
        _check(lib().crk_xdr_decode_items_batch(self.ctx.h, self.h, n, dev.data_ptr(), _stream(stream)),
               "crk_xdr_decode_items_batch")
        return dev


class ServeGraph:
    """crk_serve_graph_create / crk_graph_launch: a captured server step driven by a cursor doorbell."""

    def __init__(self, idx: Index, rings, send_rings, region_base: int, region_bytes: int, doorbell):
        n = len(rings)
        cr = (CRing * n)(*[r.c() for r in rings])
        sr = (CRing * n)(*[r.c() for r in send_rings])
        self.doorbell = doorbell
        ptr = doorbell.ptr if isinstance(doorbell, HostBuffer) else doorbell.data_ptr()
        h = vp()
        _check(lib().crk_serve_graph_create(idx.ctx.h, idx.h, n, cr, sr, region_base, region_bytes, ptr, C.byref(h)),
               "crk_serve_graph_create")
        self.h = h.value
        self.idx = idx
        idx.n_rings = n

    def launch(self, stream=None):
        _check(lib().crk_graph_launch(self.h, _stream(stream)), "crk_graph_launch")

    def close(self):
        if self.h:
            lib().crk_graph_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Server:
    """Persistent server (crk_server_start): one resident CTA serving each step the host publishes in a
    mapped pinned doorbell (ServerBell).  step() writes the windows, bumps seq and spins until the device
    publishes done_seq; it returns the per-ring results, the step status and the device service time."""

    def __init__(self, index: "Index", rings, send_rings, region_base: int, region_bytes: int, stream=None):
        self.index = index
        self.n = len(rings)
        self.buf = HostBuffer(C.sizeof(ServerBell))
        self.buf.np[:] = 0
        self.bell = ServerBell.from_address(self.buf.ptr)
        self.rings, self.send_rings = list(rings), list(send_rings)
        self.stream = stream if stream is not None else torch.cuda.Stream()
        cr = (CRing * self.n)(*[r.c() for r in self.rings])
        sr = (CRing * self.n)(*[r.c() for r in self.send_rings])
        h = vp()
        _check(lib().crk_server_start(index.ctx.h, index.h, self.n, cr, sr, region_base, region_bytes, self.buf.ptr,
                                      _stream(self.stream), C.byref(h)), "crk_server_start")
        self.h = h.value
        index.n_rings = self.n

    def step(self, windows, send_offs, timeout_s: float = 30.0) -> dict:
        """crk_server_step: the cursors written, seq bumped and done_seq awaited in C."""
        b = self.bell
        arr = u64 * self.n
        heads = arr(*[h for h, _ in windows])
        tails = arr(*[t for _, t in windows])
        offs = arr(*send_offs[:self.n])
        st = lib().crk_server_step(self.h, heads, tails, offs, int(timeout_s * 1e9))
        if st == E_CUDA:
            raise CrkError(E_CUDA, "crk_server step timed out")
        res = [dict(status=x.status, n_records=x.n_records, n_frags=x.n_frags, rec_base=x.rec_base,
                    consumed=x.consumed, reply_bytes=x.reply_bytes) for x in b.res[:self.n]]
        ph = [b.t_phase_ns[i] - b.t_begin_ns for i in range(5)]
        return {"status": b.status, "results": res, "device_ns": b.t_end_ns - b.t_begin_ns,
                "phase_end_ns": dict(zip(("setup", "scan", "parse", "plan", "move"), ph))}

    def stop(self):
        if self.h:
            h, self.h = self.h, None
            _check(lib().crk_server_stop(h), "crk_server_stop")
            # free the bell now, while no server runs: cudaFreeHost waits for the whole device, so freeing it
            # later (when the object is collected) would block behind the next persistent server forever
            self.buf.free()

    def __del__(self):
        try:
            self.stop()
        except Exception:
            pass
