"""Shared helpers for the GPU parity tests: build rings from oracle-encoded wire bytes and compare the
CUDA path's index tables with the oracle's, field by field."""
import numpy as np
import torch

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import crk, gen

PROG, VERS = gen.PROG, gen.VERS


def ocfg(strict=True, F=65536, user=None) -> O.Config:
    return O.Config(prog=PROG, vers=VERS, strict=strict, proc_h2d=gen.PROC_H2D, proc_d2h=gen.PROC_D2H,
                    frag_payload=F, user_schemas=dict(user or {}))


def ctx_for(cfg: O.Config, **kw) -> crk.Context:
    c = crk.Context(0, frag_payload=cfg.frag_payload, strict=int(cfg.strict), prog=cfg.prog, vers=cfg.vers,
                    proc_h2d=cfg.proc_h2d, proc_d2h=cfg.proc_d2h, **kw)
    for proc, items in cfg.user_schemas.items():
        c.register_schema(proc, items)
    return c


def make_ring(cap: int, host: bool = False) -> crk.Ring:
    r = crk.Ring.host(cap) if host else crk.Ring.device(cap)
    if host:
        r.host_view()[:] = 0xEE
    else:
        r.tensor().fill_(0xEE)
    return r


def ring_np(ring: crk.Ring) -> np.ndarray:
    torch.cuda.synchronize()
    hv = ring.host_view()
    return hv.copy() if hv is not None else ring.tensor().cpu().numpy()


def compare_scan(tables, ring_idx: int, ring_bytes: np.ndarray, head: int, tail: int, fpr: int, rpr: int,
                 max_record_bytes: int = 1 << 32):
    """GPU index tables of ring `ring_idx` == oracle or_frame_scan on the same bytes."""
    s = O.frame_scan(ring_bytes, head, tail, max_record_bytes, fpr, rpr)
    g = tables["rings"][ring_idx]
    assert g["status"] == s.status, (g, s.status)
    assert g["consumed"] == s.consumed
    assert g["n_records"] == len(s.recs) and g["n_frags"] == len(s.frags)
    gf = tables["frags"][ring_idx]
    if s.frags:
        assert np.array_equal(gf["phys"], np.array([f["phys"] for f in s.frags], np.uint64))
        assert np.array_equal(gf["lstart"], np.array([f["lstart"] for f in s.frags], np.uint64))
        assert np.array_equal(gf["hdr"], np.array([f["len"] | (f["last"] << 31) for f in s.frags], np.uint32))
    gr = tables["recs"][ring_idx]
    if s.recs:
        assert np.array_equal(gr["begin"], np.array([r["begin"] for r in s.recs], np.uint64))
        assert np.array_equal(gr["len"], np.array([r["len"] for r in s.recs], np.uint64))
        assert np.array_equal(gr["frag0"], np.array([r["frag0"] for r in s.recs], np.uint32))
        assert np.array_equal(gr["nfrags"], np.array([r["nfrags"] for r in s.recs], np.uint32))
    return s


def compare_parse(tables, ring_idx: int, ring_bytes: np.ndarray, scan: O.ScanResult, cfg: O.Config):
    """GPU parsed CALLs of one ring == oracle or_parse_call of each logical record."""
    P = tables["parsed"]
    base = tables["rings"][ring_idx]["rec_base"]
    calls = []
    for i in range(len(scan.recs)):
        L = O.record_logical(ring_bytes, scan, i)
        c = O.parse_call(L, cfg)
        d = base + i
        assert P["status"][d] == c.status, (i, P["status"][d], c.status)
        assert P["ring"][d] == ring_idx
        if len(L) >= 4:
            assert P["xid"][d] == c.xid
        if c.status in (O.OK, O.E_TRAILING):
            assert P["proc"][d] == c.proc and P["nitems"][d] == c.n_items
            for k in range(c.n_items):
                assert P["kind"][d, k] == c.kind[k]
                assert P["off"][d, k] == c.off[k], (i, k)
                assert P["count"][d, k] == c.count[k]
                assert P["value"][d, k] == c.value[k]
        calls.append((L, c))
    return calls


def h2d_call(xid: int, data: np.ndarray, ptr: int = 0x7F0000001000, size: int | None = None):
    return (xid, gen.PROC_H2D, [(O.K_U64, ptr), (O.K_OPAQUE_VAR, data.tobytes()),
                                (O.K_U64, len(data) if size is None else size)])


def d2h_call(xid: int, ptr: int, size: int):
    return (xid, gen.PROC_D2H, [(O.K_U64, ptr), (O.K_U64, size)])
