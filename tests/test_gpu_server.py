"""GPU parity of the persistent server (crk_server_*) against the oracle's serve
step (oracle/oracle.c or_serve), bit-exact: several steps through one resident kernel, each appending a
batch of calls (HtoD / DtoH memcpys, control calls, every error kind serve reports) to every ring.

While a server runs, nothing here may synchronise the whole device (its kernel never ends until stop):
results come from the doorbell block, memory is read with stream-ordered copies."""
import os

import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import crk, gen
from tests.gpu_util import compare_parse, compare_scan, ctx_for, d2h_call, h2d_call, make_ring, ocfg

pytestmark = [pytest.mark.gpu, pytest.mark.timeout(300)]
# CRK_FUZZ_SEED shifts every seed (longer fuzz campaigns: tools/gpu_tests.sh with the variable set)
SEED = int(os.environ.get("CRK_FUZZ_SEED", "0"))

if not torch.cuda.is_available():
    pytest.skip("needs a GPU", allow_module_level=True)


def ring_bytes(ring: crk.Ring) -> np.ndarray:
    hv = ring.host_view()
    if hv is not None:
        return hv.copy()
    return ring.tensor().cpu().numpy()  # stream-ordered copy, no device-wide synchronisation


def batch(g, step: int, ring: int, base: int, region_bytes: int, host_region: np.ndarray, cfg, F: int):
    """Wire bytes of one step's calls on one ring: small HtoD / DtoH memcpys, a control call of a
    registered proc, and (some steps) error records."""
    wire = b""
    for i in range(int(g.integers(1, 6))):
        xid = (step << 20) | (ring << 12) | i
        kind = int(g.integers(0, 3))
        if kind == 0:  # destinations: a private slot of the region's lower half (reading R18: disjoint)
            size = int(g.integers(0, 20000))
            off = (ring * 6 + i) * 20480 + int(g.integers(0, 16))
            data = gen.random_bytes((step * 131 + ring * 17 + i) & 0xFFFFFFFF, size)
            c = h2d_call(xid, data, base + off)
        elif kind == 1:  # sources: the upper half, never written
            size = int(g.integers(0, 40000))
            off = region_bytes // 2 + int(g.integers(0, region_bytes // 2 - size))
            c = d2h_call(xid, base + off, size)
        else:
            c = (xid, 33, [(O.K_U32, int(g.integers(0, 1 << 32))), (O.K_I32_VAR, gen.random_elems(g, np.int32, 17))])
        wire += O.encode_call(*c, cfg, F=F)
    if step % 3 == 2:  # a duplicate xid, a pointer outside the region, a wrong program version
        wire += O.encode_call(*h2d_call((step << 20) | (ring << 12), np.zeros(8, np.uint8), base), cfg, F=F)
        wire += O.encode_call(*d2h_call(0xE0000000 + step, base + region_bytes, 16), cfg, F=F)
        wire += O.frame(O.call_header(0xE2000000 + step, gen.PROG, 3, 1), 100)
    return wire


@pytest.mark.parametrize("host", [False, True])
def test_server_steps_match_oracle(host):
    F = 4096
    cfg = ocfg(F=F, user={33: [O.K_U32, O.K_I32_VAR]})
    ctx = ctx_for(cfg)
    n_rings, cap, scap = 3, 1 << 18, 1 << 18
    region_bytes = 1 << 20
    region = torch.zeros(region_bytes, dtype=torch.uint8, device="cuda")
    base = region.data_ptr()
    g = gen.rng(0x5E + SEED)
    host_region = gen.random_bytes(0x5E5E, region_bytes).copy()
    region.copy_(torch.from_numpy(host_region))
    rings = [crk.Ring.host(cap) if host else crk.Ring.device(cap) for _ in range(n_rings)]
    sends = [crk.Ring.host(scap) if host else crk.Ring.device(scap) for _ in range(n_rings)]
    idx = ctx.index(n_rings, 1 << 12, 3 * 64)
    torch.cuda.synchronize()
    srv = crk.Server(idx, rings, sends, base, region_bytes)
    try:
        tails = [cap - 5000 + 97 * r for r in range(n_rings)]  # windows cross the wrap on later steps
        send_offs = [scap - 3000 + 11 * r for r in range(n_rings)]
        for step in range(8):
            heads = list(tails)
            for r in range(n_rings):
                w = batch(g, step, r, base, region_bytes, host_region, cfg, F)
                rings[r].write(tails[r], w)
                tails[r] += len(w)
            if step == 5:  # a truncated window: the last record is incomplete
                tails[1] -= 3
            before = [ring_bytes(r) for r in rings]
            out = srv.step(list(zip(heads, tails)), send_offs)
            want = O.serve([(b, h, t) for b, h, t in zip(before, heads, tails)], cfg, host_region, base,
                           [scap] * n_rings, send_offs, max_frags_per_ring=(1 << 12) // n_rings,
                           max_records_per_ring=64)
            assert out["status"] == O.OK
            for r in range(n_rings):
                res = out["results"][r]
                assert res["status"] == want["scan_status"][r], (step, r, res)
                assert res["consumed"] == want["consumed"][r], (step, r)
                assert res["reply_bytes"] == want["reply_bytes"][r], (step, r)
                n = want["reply_bytes"][r]
                got = sends[r].read(send_offs[r], n)
                exp = bytes(np.roll(want["send"][r], -(send_offs[r] % scap))[:n])
                assert got == exp, (step, r)
            assert np.array_equal(region.cpu().numpy(), host_region), step
            for r in range(n_rings):
                tails[r] = want["consumed"][r] if step == 5 and r == 1 else tails[r]
                send_offs[r] += want["reply_bytes"][r]
    finally:
        srv.stop()


def test_server_rejects_bad_window_and_stops():
    cfg = ocfg()
    ctx = ctx_for(cfg)
    region = torch.zeros(1 << 16, dtype=torch.uint8, device="cuda")
    ring, send = crk.Ring.device(1 << 12), crk.Ring.device(1 << 12)
    idx = ctx.index(1, 64, 16)
    torch.cuda.synchronize()
    srv = crk.Server(idx, [ring], [send], region.data_ptr(), region.numel())
    try:
        out = srv.step([(100, 50)], [0])  # tail < head
        assert out["status"] == crk.E_ARG and out["results"][0]["n_records"] == 0
        w = O.encode_call(*h2d_call(9, np.arange(100, dtype=np.uint8), region.data_ptr() + 8), cfg)
        ring.write(0, w)
        out = srv.step([(0, len(w))], [0])
        assert out["status"] == crk.OK and out["results"][0]["status"] == crk.OK
        assert out["results"][0]["consumed"] == len(w) and out["device_ns"] > 0
        assert np.array_equal(region[8:108].cpu().numpy(), np.arange(100, dtype=np.uint8))
    finally:
        srv.stop()
    torch.cuda.synchronize()  # the kernel has exited


def test_server_capacity_limits():
    ctx = ctx_for(ocfg())
    ring, send = crk.Ring.device(1 << 12), crk.Ring.device(1 << 12)
    with pytest.raises(crk.CrkError):
        crk.Server(ctx.index(1, 1 << 12, 2048), [ring], [send], 0, 0)  # > 1024 records


@pytest.mark.parametrize("fused", [False, True])
def test_serve_steps_across_the_wrap_match_oracle(fused):
    """The same multi-step stream through crk_serve launches (windows and send cursors crossing the ring
    wrap, error records, a truncated window), with the separate scan / parse / plan kernels and with the
    fused single-CTA front end."""
    F = 4096
    cfg = ocfg(F=F, user={33: [O.K_U32, O.K_I32_VAR]})
    ctx = ctx_for(cfg, fused_front_max_records=1024 if fused else 0, fused_front_max_window=1 << 30)
    n_rings, cap, scap = 3, 1 << 18, 1 << 18
    region_bytes = 1 << 20
    region = torch.zeros(region_bytes, dtype=torch.uint8, device="cuda")
    base = region.data_ptr()
    g = gen.rng(0x5F + SEED)
    host_region = gen.random_bytes(0x5F5F, region_bytes).copy()
    region.copy_(torch.from_numpy(host_region))
    rings = [crk.Ring.device(cap) for _ in range(n_rings)]
    sends = [crk.Ring.device(scap) for _ in range(n_rings)]
    idx = ctx.index(n_rings, 1 << 12, 3 * 64)
    tails = [cap - 5000 + 97 * r for r in range(n_rings)]
    send_offs = [scap - 3000 + 11 * r for r in range(n_rings)]
    for step in range(8):
        heads = list(tails)
        for r in range(n_rings):
            w = batch(g, step, r, base, region_bytes, host_region, cfg, F)
            rings[r].write(tails[r], w)
            tails[r] += len(w)
        if step == 5:
            tails[1] -= 3
        before = [ring_bytes(r) for r in rings]
        idx.serve([(rg, h, t) for rg, h, t in zip(rings, heads, tails)], sends, send_offs, base, region_bytes)
        torch.cuda.synchronize()
        want = O.serve([(b, h, t) for b, h, t in zip(before, heads, tails)], cfg, host_region, base,
                       [scap] * n_rings, send_offs, max_frags_per_ring=(1 << 12) // n_rings, max_records_per_ring=64)
        res = idx.ring_results(n_rings)
        for r in range(n_rings):
            assert res[r]["status"] == want["scan_status"][r], (step, r, res[r])
            assert res[r]["consumed"] == want["consumed"][r], (step, r)
            assert res[r]["reply_bytes"] == want["reply_bytes"][r], (step, r)
            n = want["reply_bytes"][r]
            exp = bytes(np.roll(want["send"][r], -(send_offs[r] % scap))[:n])
            assert sends[r].read(send_offs[r], n) == exp, (step, r)
        assert np.array_equal(region.cpu().numpy(), host_region), step
        for r in range(n_rings):
            tails[r] = want["consumed"][r] if step == 5 and r == 1 else tails[r]
            send_offs[r] += want["reply_bytes"][r]


def test_servers_back_to_back_on_one_context():
    """A persistent server stopped and another started on the same context and index (the binding frees each
    bell at stop: freeing pinned memory later would wait for the next running server forever)."""
    import gc
    gc.collect()  # garbage from earlier tests (pinned rings of a failed one) freed before any server runs
    torch.cuda.synchronize()
    cfg = ocfg()
    ctx = ctx_for(cfg)
    region = torch.zeros(1 << 16, dtype=torch.uint8, device="cuda")
    base = region.data_ptr()
    ring = make_ring(1 << 14)
    payload = gen.random_bytes(9, 4096)
    w = O.encode_call(7, gen.PROC_H2D, [(O.K_U64, base + 64), (O.K_OPAQUE_VAR, payload.tobytes()),
                                        (O.K_U64, 4096)], cfg)
    ring.write(0, w)
    send = make_ring(1 << 12)
    idx = ctx.index(1, 64, 16)
    for rep in range(3):
        srv = crk.Server(idx, [ring], [send], base, region.numel())
        gc.collect()  # the previous server object goes away while this one runs
        out = srv.step([(0, len(w))], [0], timeout_s=20)
        assert out["results"][0]["status"] == O.OK and out["results"][0]["reply_bytes"] == 32
        srv.stop()
    assert region[64:64 + 4096].cpu().numpy().tobytes() == payload.tobytes()


def _mover_jobs(ctx) -> int:
    """The context's planned job count (scratch counter 1; the lean path leaves 0 for the mover)."""
    return ctx.debug_counters()[1]


@pytest.mark.parametrize("mode,host,strict,F", [("server", False, True, 100), ("server", False, False, 4096),
                                                ("server", True, True, 1024), ("serve", False, True, 100),
                                                ("serve", True, False, 1024)])
def test_lean_steps_match_oracle(mode, host, strict, F):
    """Steps of well-formed memcpy CALLs only (single- and multi-fragment) -- the lean path (one warp over a shared-
    memory copy of the windows) of the persistent server and of crk_serve's fused front end -- against the oracle: ring
    results, reply bytes (framed with F, here smaller than most replies), destination bytes, and the index tables
    the general phases would have written (fragment / record tables vs or_frame_scan, parsed CALLs vs
    or_parse_call, serve decisions vs or_serve)."""
    cfg = ocfg(strict=strict, F=F, user={33: [O.K_U32, O.K_I32_VAR], 34: [O.K_U64, O.K_OPAQUE_FIX | (13 << 8)]})
    ctx = ctx_for(cfg, fused_front_max_records=1024, fused_front_max_window=1 << 30, lean_backoff=0)
    n_rings, cap, scap = 3, 1 << 16, 1 << 18
    region_bytes = 1 << 20
    region = torch.zeros(region_bytes, dtype=torch.uint8, device="cuda")
    base = region.data_ptr()
    g = gen.rng(0x1EA + F + 2 * strict + host + SEED)
    host_region = gen.random_bytes(0x1EA1, region_bytes).copy()
    region.copy_(torch.from_numpy(host_region))
    rings = [crk.Ring.host(cap) if host else crk.Ring.device(cap) for _ in range(n_rings)]
    sends = [crk.Ring.host(scap) if host else crk.Ring.device(scap) for _ in range(n_rings)]
    idx = ctx.index(n_rings, 3 * 64, 3 * 32)
    torch.cuda.synchronize()
    srv = crk.Server(idx, rings, sends, base, region_bytes) if mode == "server" else None
    lean = 0
    try:
        tails = [cap - 3000 + 37 * r for r in range(n_rings)]  # windows cross the wrap
        send_offs = [scap - 2000 + 4 * r for r in range(n_rings)]
        for step in range(12):
            heads = list(tails)
            for r in range(n_rings):
                wire = b""
                for i in range(int(g.integers(0, 5))):
                    xid = (step << 16) | (r << 8) | i
                    k = int(g.integers(0, 5 if mode == "server" else 4))
                    if k == 4:  # a control call (the server's lean path takes registered procedures too)
                        if g.integers(0, 2):
                            c = (xid, 33, [(O.K_U32, int(g.integers(0, 1 << 32))),
                                           (O.K_I32_VAR, gen.random_elems(g, np.int32, int(g.integers(0, 40))))])
                        else:
                            c = (xid, 34, [(O.K_U64, int(g.integers(0, 1 << 62))),
                                           (O.K_OPAQUE_FIX, gen.random_bytes(xid & 0xFFFF, 13).tobytes())])
                    elif k < 2:  # HtoD to a private slot of the lower half, any alignment
                        data = gen.random_bytes((step * 7 + r * 3 + i) & 0xFFFF, int(g.integers(0, 2500)))
                        c = h2d_call(xid, data, base + (r * 4 + i) * 4096 + int(g.integers(0, 64)))
                    else:  # DtoH from the upper half
                        size = int(g.integers(0, 5000))
                        c = d2h_call(xid, base + region_bytes // 2 + int(g.integers(0, region_bytes // 2 - size)), size)
                    # one fragment per CALL, or several (the first one always holds the fixed-layout head)
                    wire += O.encode_call(*c, cfg, F=int(g.choice([1 << 16, 1000, 256])))
                rings[r].write(tails[r], wire)
                tails[r] += len(wire)
            before = [ring_bytes(rg) for rg in rings]
            if srv:
                out = srv.step(list(zip(heads, tails)), send_offs)
                assert out["status"] == O.OK
                ph = list(out["phase_end_ns"].values())
                lean += ph[1] == ph[2] == ph[3] == ph[4]  # the lean path stamps its phases at once
            else:
                idx.serve([(rg, h, t) for rg, h, t in zip(rings, heads, tails)], sends, send_offs, base,
                          region_bytes)
                torch.cuda.synchronize()
                out = {"results": idx.ring_results(n_rings)}
                lean += _mover_jobs(ctx) == 0 and sum(r["n_records"] for r in out["results"]) > 0
            want = O.serve([(b, h, t) for b, h, t in zip(before, heads, tails)], cfg, host_region, base,
                           [scap] * n_rings, send_offs, max_frags_per_ring=64, max_records_per_ring=32)
            for r in range(n_rings):
                res = out["results"][r]
                assert res["status"] == want["scan_status"][r] == O.OK, (step, r, res)
                assert res["consumed"] == want["consumed"][r] == tails[r], (step, r)
                assert res["reply_bytes"] == want["reply_bytes"][r], (step, r)
                n = want["reply_bytes"][r]
                exp = bytes(np.roll(want["send"][r], -(send_offs[r] % scap))[:n])
                assert sends[r].read(send_offs[r], n) == exp, (step, r)
            assert np.array_equal(region.cpu().numpy(), host_region), step
            T = idx.tables(n_rings, sync=srv is None)
            for r in range(n_rings):
                s = compare_scan(T, r, before[r], heads[r], tails[r], 64, 32)
                compare_parse(T, r, before[r], s, cfg)
            P = T["parsed"]
            assert [x["status"] for x in want["records"]] == list(P["serve_status"]), step
            assert [x["reply_err"] for x in want["records"]] == list(P["serve_reply_err"]), step
            assert [x["reply_wire"] for x in want["records"]] == list(P["serve_reply_wire"]), step
            assert [x["reply_off"] for x in want["records"]] == list(P["serve_reply_off"]), step
            for r in range(n_rings):
                send_offs[r] += want["reply_bytes"][r]
    finally:
        if srv:
            srv.stop()
    assert lean >= 5, lean  # most steps took the lean path


@pytest.mark.parametrize("lean_steps,backoff", [(0, 16), (1, 16)])
def test_lean_switch_and_backoff(lean_steps, backoff):
    """crk_config.lean_steps = 0 keeps every step on the general phases; with the back-off, a step the lean path
    cannot take (a control call) makes the next `backoff` steps skip the attempt, after which it is tried again.
    Results equal the oracle's either way."""
    cfg = ocfg(F=4096, user={33: [O.K_U32]})
    ctx = ctx_for(cfg, lean_steps=lean_steps, lean_backoff=backoff)
    region = torch.zeros(1 << 16, dtype=torch.uint8, device="cuda")
    base = region.data_ptr()
    ring, send = crk.Ring.device(1 << 16), crk.Ring.device(1 << 16)
    idx = ctx.index(1, 64, 16)
    data = gen.random_bytes(5, 1000)
    memcpy = O.encode_call(*h2d_call(1, data, base + 64), cfg)
    control = O.encode_call(2, 33, [(O.K_U32, 7)], cfg)
    took = []
    head = 0
    for step in range(2 + backoff + 1):
        w = control if step == 1 else memcpy
        ring.write(head, w)
        idx.serve([(ring, head, head + len(w))], [send], [0], base, region.numel())
        torch.cuda.synchronize()
        res = idx.ring_results(1)[0]
        assert res["status"] == O.OK and res["consumed"] == head + len(w)
        took.append(ctx.debug_counters()[1] == 0)  # the lean path leaves the mover an empty plan
        head += len(w)
    assert np.array_equal(region[64:1064].cpu().numpy(), data)
    if lean_steps == 0:
        assert not any(took)
    else:  # lean, the control call (general), `backoff` general steps, lean again
        assert took == [True, False] + [False] * backoff + [True], took
