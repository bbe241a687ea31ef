"""Per-config measurements beside the bench headline.

Device-resident rings, CUDA-event timing on the launching stream after warm-up; every config checks its
output against the generator's values.  Writes one JSON object (stdout).

  C1   one CALL (4 KiB opaque + 1,024 int32): latency of scan+parse -> memcpy decode -> int32 decode, and
       131,072 back-to-back records: records/s and GB/s of scan+parse+batch decode
  C2   matrixMul transfers (A, B HtoD; C DtoH) served as one batch: microseconds
  C3   bandwidth sweep: HtoD (scan+parse+decode) and DtoH (reply encode) GB/s per size, buffers rotated
       over >= 256 MiB so repeated runs do not hit L2
  C4   256 MiB typed-array stress: decode GB/s (all items, regular and irregular framing)
  NEXT-1  one 1 GiB memcpy striped over 16 / 4 rings (stripe CALLs, reading R22: one reply for the memcpy) vs one
          1 GiB CALL on one ring and 16 separate 64 MiB CALLs, each served as one batch
  NEXT-2  gen.cusolver_endpoint (100 iterations of A 900x900 f64 + b HtoD, x DtoH; 1 and 4 client streams) and
          gen.histogram_endpoint (64 MiB HtoD, 256-bin result DtoH), served by crk_serve
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_sc_eilingkkflm23_b200 import build, crk, gen  # noqa: E402

MiB, GiB = 1 << 20, 1 << 30
dev = torch.device("cuda:0")
# crk_config overrides for every context of the suite, e.g. SUITE_CTX=scan_threads=512
CTX_KW = {k: int(v, 0) for k, v in (kv.split("=") for kv in os.environ.get("SUITE_CTX", "").split(",") if kv)}


def Ctx():
    return crk.Context(0, **CTX_KW)


def timed(fn, reps, warm=3):
    for _ in range(warm):
        fn(0)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for i in range(reps):
        fn(i)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps  # ms


_flush = None


def timed_cold(fn, reps, warm=2):
    """Mean ms of fn over reps runs, each timed alone after writing a buffer larger than L2."""
    global _flush
    if _flush is None:
        _flush = torch.empty(512 * MiB, dtype=torch.uint8, device=dev)
    for _ in range(warm):
        fn(0)
    tot = 0.0
    for i in range(reps):
        _flush.fill_(i & 0xFF)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn(i)
        e1.record()
        torch.cuda.synchronize()
        tot += e0.elapsed_time(e1)
    return tot / reps


def next_pow2(x):
    return 1 << max(8, (x - 1).bit_length())


def c1(ctx):
    ctx.register_schema(gen.PROC_C1, gen.C1_SCHEMA)
    c = gen.c1_call(xid=1)
    data = torch.from_numpy(c.items[1][1]).to(dev)
    ints = torch.from_numpy(c.items[3][1]).to(dev)
    items = [(crk.K_U64, c.items[0][1]), (crk.K_OPAQUE_VAR, data), (crk.K_U64, 4096), (crk.K_I32_VAR, ints)]
    ring = crk.Ring.device(1 << 14)
    w = ctx.encode_call(1, gen.PROC_C1, items, ring, 0)
    idx = ctx.index(1, 64, 16)
    dst = torch.empty(4096, dtype=torch.uint8, device=dev)
    out = torch.empty(1024, dtype=torch.int32, device=dev)
    st = torch.zeros(2, dtype=torch.int32, device=dev)
    cnt = torch.zeros(2, dtype=torch.int64, device=dev)

    def one(_):
        idx.frame_scan([(ring, 0, w)])
        idx.decode_opaque(1, 1, dst, 4096, cnt[0:1], st[0:1])
        idx.decode_array("i32", 1, 3, out, 1024, cnt[1:2], st[1:2])

    lat_ms = timed(one, 200)
    ok = bool(torch.equal(dst, data) and torch.equal(out, ints) and (st == 0).all())
    # the same three calls captured once as a CUDA graph and replayed: device-side latency without the
    # Python / ctypes issue cost of the loop above (which bounds it when launches are this short)
    g = torch.cuda.CUDAGraph()
    cs = torch.cuda.Stream()
    cs.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(cs):
        one(0)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=cs):
            one(0)
    torch.cuda.current_stream().wait_stream(cs)
    dst.zero_(); out.zero_(); st.fill_(-1)
    lat_graph_ms = timed(lambda _: g.replay(), 200)
    ok &= bool(torch.equal(dst, data) and torch.equal(out, ints) and (st == 0).all())
    # 131,072 back-to-back records
    n = 131072
    big = crk.Ring.device(next_pow2(n * w + 4096))
    big.tensor()[:w].copy_(ring.tensor()[:w])
    reps = torch.arange(n, device=dev, dtype=torch.int64)
    body = big.tensor()[:w].clone()
    view = big.tensor()[:n * w].view(n, w)
    view.copy_(body.unsqueeze(0).expand(n, w))
    xids = (torch.arange(n, dtype=torch.int64) + 0x100000).to(torch.int32)
    xb = xids.numpy().astype(">u4").view(np.uint8).reshape(n, 4)
    view[:, 4:8].copy_(torch.from_numpy(xb.copy()).to(dev))  # distinct xids
    idx2 = ctx.index(1, n + 16, n + 16)
    dsts = torch.empty((n, 4096), dtype=torch.uint8, device=dev)
    outs = torch.empty((n, 1024), dtype=torch.int32, device=dev)
    sts = torch.zeros(2 * n, dtype=torch.int32, device=dev)
    reqs = []
    for i in range(n):
        reqs.append((int(xids[i]), 1, crk.K_OPAQUE_VAR, dsts[i].data_ptr(), 4096, None, sts.data_ptr() + 8 * i))
        reqs.append((int(xids[i]), 3, crk.K_I32_VAR, outs[i].data_ptr(), 1024, None, sts.data_ptr() + 8 * i + 4))
    arr = (crk.ItemReq * len(reqs))(*[crk.ItemReq(a, b, c_, 0, d, e, f, g) for a, b, c_, d, e, f, g in reqs])
    dreq = torch.frombuffer(bytearray(arr), dtype=torch.uint8).to(dev)

    def batch(_):
        idx2.frame_scan([(big, 0, n * w)])
        crk._check(crk.lib().crk_xdr_decode_items_batch(ctx.h, idx2.h, len(reqs), dreq.data_ptr(),
                                                         torch.cuda.current_stream().cuda_stream), "batch")

    bms = timed(batch, 5, warm=1)
    ok2 = bool((sts == 0).all() and torch.equal(dsts[n - 1], data) and torch.equal(outs[12345], ints))
    return {"latency_us": round(lat_ms * 1e3, 2), "latency_graph_us": round(lat_graph_ms * 1e3, 2), "ok": ok,
            "note": "one record: crk_rpc_frame_scan (scan+parse) + crk_xdr_decode_opaque + crk_xdr_decode_array_i32",
            "batch_records": n, "batch_ms": round(bms, 3), "records_per_s": round(n / bms * 1e3),
            "batch_payload_gbs": round(n * 8192 / bms / 1e6, 1), "batch_ok": ok2}


def serve_latency(ctx):
    """One 4 KiB HtoD CALL served per step (scan, parse, plan, mover, reply): crk_serve launches versus the
    same step replayed from a CUDA graph whose cursors come from a doorbell."""
    region = torch.zeros(1 << 20, dtype=torch.uint8, device=dev)
    base = region.data_ptr()
    data = torch.from_numpy(gen.random_bytes(0xC1, 4096)).to(dev)
    ring = crk.Ring.device(1 << 14)
    w = ctx.encode_call(7, gen.PROC_H2D, [(crk.K_U64, base + 4096), (crk.K_OPAQUE_VAR, data), (crk.K_U64, 4096)],
                        ring, 0)
    send = crk.Ring.device(1 << 12)
    idx = ctx.index(1, 64, 16)
    # (host-bound: a long warm-up, or the first entry of the suite pays the host's ramp -- 22 vs 15 us)
    us_launch = timed(lambda _: idx.serve([(ring, 0, w)], [send], [0], base, region.numel()), 500, warm=300) * 1e3
    bell = torch.tensor([0, w, 0], dtype=torch.int64, device=dev)
    g = idx.serve_graph([ring], [send], base, region.numel(), bell)
    us_graph = timed(lambda _: g.launch(), 500) * 1e3
    ok = bool(torch.equal(region[4096:8192], data)) and idx.ring_results(1)[0]["reply_bytes"] == 32
    g.close()
    # one control call of a registered procedure per step, graph replay (the server's NEXT3 control call)
    ctx.register_schema(60, [crk.K_U64, crk.K_U32, crk.K_U32, crk.K_OPAQUE_VAR])
    ring4 = crk.Ring.device(1 << 12)
    w4 = ctx.encode_call(9, 60, [(crk.K_U64, 0x7F00DEADBEEF), (crk.K_U32, 148), (crk.K_U32, 256),
                                 (crk.K_OPAQUE_VAR, data[:64])], ring4, 0)
    bell4 = torch.tensor([0, w4, 0], dtype=torch.int64, device=dev)
    g4 = idx.serve_graph([ring4], [send], base, region.numel(), bell4)
    us_ctl = timed(lambda _: g4.launch(), 500) * 1e3
    res4 = idx.ring_results(1)[0]
    ok4 = res4["status"] == 0 and res4["n_records"] == 1 and res4["reply_bytes"] == 0
    g4.close()
    return {"serve_launches_us": round(us_launch, 2), "serve_graph_us": round(us_graph, 2), "ok": ok,
            "control_call_graph_us": round(us_ctl, 2), "control_ok": bool(ok4)}


def server_latency(ctx, reps=2000):
    """Persistent server (crk_server): one 4 KiB HtoD CALL per step, published through a mapped doorbell;
    host round trip (write cursors, bump seq, spin on done_seq) and the device's service time per step.
    Then the C2 matrixMul batch (A, B HtoD; C DtoH) as one step."""
    import time
    region = torch.zeros(4 * MiB, dtype=torch.uint8, device=dev)
    base = region.data_ptr()
    data = torch.from_numpy(gen.random_bytes(0xC1, 4096)).to(dev)
    ring = crk.Ring.device(1 << 14)
    w = ctx.encode_call(7, gen.PROC_H2D, [(crk.K_U64, base + 4096), (crk.K_OPAQUE_VAR, data), (crk.K_U64, 4096)],
                        ring, 0)
    send = crk.Ring.device(1 << 21)
    idx = ctx.index(1, 64, 16)
    # the C2 matrixMul batch, encoded before any server owns the context
    A, B, Cm = gen.c2_matrices()
    a, b = torch.from_numpy(A.view(np.uint8)).to(dev), torch.from_numpy(B.view(np.uint8)).to(dev)
    ring2 = crk.Ring.device(1 << 21)
    cur = ctx.encode_call(1, gen.PROC_H2D, [(crk.K_U64, base), (crk.K_OPAQUE_VAR, a), (crk.K_U64, a.numel())],
                          ring2, 0)
    cur += ctx.encode_call(2, gen.PROC_H2D, [(crk.K_U64, base + MiB), (crk.K_OPAQUE_VAR, b), (crk.K_U64, b.numel())],
                           ring2, cur)
    cur += ctx.encode_call(3, gen.PROC_D2H, [(crk.K_U64, base + 3 * MiB), (crk.K_U64, Cm.nbytes)], ring2, cur)
    # twelve 4 KiB HtoD CALLs in one step (a server collecting several clients' small calls)
    ring3 = crk.Ring.device(1 << 16)
    cur3 = 0
    for i in range(12):
        cur3 += ctx.encode_call(100 + i, gen.PROC_H2D, [(crk.K_U64, base + 2 * MiB + 4096 * i), (crk.K_OPAQUE_VAR, data),
                                                        (crk.K_U64, 4096)], ring3, cur3)
    # one control call of a registered procedure (a kernel launch's handle, grid size and a 64-byte parameter block)
    ctx.register_schema(60, [crk.K_U64, crk.K_U32, crk.K_U32, crk.K_OPAQUE_VAR])
    ring4 = crk.Ring.device(1 << 12)
    params = torch.from_numpy(gen.random_bytes(0x60, 64)).to(dev)
    cur4 = ctx.encode_call(9, 60, [(crk.K_U64, 0x7F00DEADBEEF), (crk.K_U32, 148), (crk.K_U32, 256),
                                   (crk.K_OPAQUE_VAR, params)], ring4, 0)
    torch.cuda.synchronize()
    srv = crk.Server(idx, [ring], [send], base, region.numel())
    try:
        rt, dv, ph = [], [], []
        for i in range(reps):
            t0 = time.perf_counter_ns()
            out = srv.step([(0, w)], [0])
            rt.append(time.perf_counter_ns() - t0)
            dv.append(out["device_ns"])
            ph.append(list(out["phase_end_ns"].values()))
        ok = out["results"][0]["status"] == 0 and out["results"][0]["reply_bytes"] == 32
        # the same step timed around the C call alone (crk_server_step: cursors, seq, spin on done_seq)
        import ctypes as C
        u64a = C.c_uint64 * 1
        hs, ts, so = u64a(0), u64a(w), u64a(0)
        crt = []
        for i in range(reps):
            t0 = time.perf_counter_ns()
            st = crk.lib().crk_server_step(srv.h, hs, ts, so, 10 ** 9)
            crt.append(time.perf_counter_ns() - t0)
            ok &= st == 0
    finally:
        srv.stop()
    ok &= bool(torch.equal(region[4096:8192], data))  # device allocations wait for a running server
    idx2 = ctx.index(1, 1024, 16)
    srv2 = crk.Server(idx2, [ring2], [send], base, region.numel())
    try:
        c2dv = []
        for i in range(50):
            out2 = srv2.step([(0, cur)], [0])
            c2dv.append(out2["device_ns"])
        ok2 = out2["results"][0]["status"] == 0
    finally:
        srv2.stop()
    ok2 &= bool(torch.equal(region[:a.numel()], a))
    srv3 = crk.Server(ctx.index(1, 64, 16), [ring3], [send], base, region.numel())
    try:
        m12 = []
        for i in range(200):
            out3 = srv3.step([(0, cur3)], [0])
            m12.append(out3["device_ns"])
        ok3 = out3["results"][0]["status"] == 0 and out3["results"][0]["n_records"] == 12
    finally:
        srv3.stop()
    ok3 &= all(bool(torch.equal(region[2 * MiB + 4096 * i:2 * MiB + 4096 * (i + 1)], data)) for i in range(12))
    srv4 = crk.Server(ctx.index(1, 64, 16), [ring4], [send], base, region.numel())
    try:
        mc = []
        for i in range(500):
            out4 = srv4.step([(0, cur4)], [0])
            mc.append(out4["device_ns"])
        ok4 = out4["results"][0]["status"] == 0 and out4["results"][0]["n_records"] == 1
    finally:
        srv4.stop()
    t12 = float(np.median(m12))
    return {"one_record_c_roundtrip_us_median": round(float(np.median(crt)) / 1e3, 2),
            "one_record_c_roundtrip_us_p99": round(float(np.percentile(crt, 99)) / 1e3, 2),
            "one_record_roundtrip_us_median": round(float(np.median(rt)) / 1e3, 2),
            "one_record_device_us_median": round(float(np.median(dv)) / 1e3, 2),
            "one_record_roundtrip_us_p99": round(float(np.percentile(rt, 99)) / 1e3, 2), "ok": bool(ok),
            "one_record_phase_end_us_median": dict(zip(("setup", "scan", "parse", "plan", "move"),
                                                      [round(float(x) / 1e3, 2) for x in np.median(ph, axis=0)])),
            "c2_batch_device_us_median": round(float(np.median(c2dv)) / 1e3, 2), "c2_ok": bool(ok2),
            "twelve_4KiB_calls_device_us_median": round(t12 / 1e3, 2),
            "twelve_4KiB_calls_gbs": round(12 * 4096 / t12, 2), "twelve_ok": bool(ok3),
            "control_call_device_us_median": round(float(np.median(mc)) / 1e3, 2), "control_ok": bool(ok4)}


def c2(ctx):
    A, B, C = gen.c2_matrices()
    region = torch.zeros(4 * MiB, dtype=torch.uint8, device=dev)
    base = region.data_ptr()
    a = torch.from_numpy(A.view(np.uint8)).to(dev)
    b = torch.from_numpy(B.view(np.uint8)).to(dev)
    region[3 * MiB:3 * MiB + C.nbytes].copy_(torch.from_numpy(C.view(np.uint8)))
    ring = crk.Ring.device(1 << 21)
    cur = 0
    cur += ctx.encode_call(1, gen.PROC_H2D, [(crk.K_U64, base), (crk.K_OPAQUE_VAR, a), (crk.K_U64, a.numel())], ring, cur)
    cur += ctx.encode_call(2, gen.PROC_H2D, [(crk.K_U64, base + MiB), (crk.K_OPAQUE_VAR, b), (crk.K_U64, b.numel())],
                           ring, cur)
    cur += ctx.encode_call(3, gen.PROC_D2H, [(crk.K_U64, base + 3 * MiB), (crk.K_U64, C.nbytes)], ring, cur)
    send = crk.Ring.device(1 << 21)
    idx = ctx.index(1, 1024, 16)
    ms = timed(lambda _: idx.serve([(ring, 0, cur)], [send], [0], base, region.numel()), 200)
    ok = bool(torch.equal(region[:a.numel()], a) and torch.equal(region[MiB:MiB + b.numel()], b))
    res = idx.ring_results(1)[0]
    ok &= res["reply_bytes"] == crk.wire_size_d2h(C.nbytes, 0) + 2 * crk.wire_size_d2h(0, 1)
    return {"us": round(ms * 1e3, 2), "bytes": int(A.nbytes + B.nbytes + C.nbytes), "wire_in": cur,
            "reply_wire": res["reply_bytes"], "gbs": round((A.nbytes + B.nbytes + C.nbytes) / ms / 1e6, 2), "ok": ok}


def c3(ctx, logs=(12, 14, 16, 18, 20, 22, 24, 26, 27, 28, 29, 30)):
    out = []
    for lg in logs:
        n = 1 << lg
        payload = torch.from_numpy(gen.c3_payload(lg)).to(dev)
        one = crk.Ring.device(next_pow2(n + 4 * (n // 65536 + 2) + 64))
        w = ctx.encode_call(lg, gen.PROC_H2D, [(crk.K_U64, 0), (crk.K_OPAQUE_VAR, payload), (crk.K_U64, n)], one, 0)
        copies = max(1, min(64, (256 * MiB) // max(w, 1)))
        rings = [one] + [crk.Ring.device(one.cap) for _ in range(copies - 1)]
        for r in rings[1:]:
            r.tensor()[:w].copy_(one.tensor()[:w])
        dsts = [torch.empty(n, dtype=torch.uint8, device=dev) for _ in range(copies)]
        idx = ctx.index(1, n // 65536 + 16, 4)
        st = torch.zeros(1, dtype=torch.int32, device=dev)

        def h2d(i):
            k = i % copies
            idx.frame_scan([(rings[k], 0, w)])
            idx.decode_memcpy_h2d(lg, dsts[k], n, st)

        reps = max(10, min(400, (GiB // n)))
        ms = timed(h2d, reps)
        ok = bool(torch.equal(dsts[(reps - 1) % copies], payload)) and st.item() == 0
        outs = [crk.Ring.device(next_pow2(crk.wire_size_d2h(n, 0) + 64)) for _ in range(copies)]
        srcs = [payload] + [payload.clone() for _ in range(copies - 1)]
        wd = crk.wire_size_d2h(n, 0)
        ms_d = timed(lambda i: ctx.encode_memcpy_d2h(lg, srcs[i % copies], 0, outs[i % copies], 0), reps)
        out.append({"log2n": lg, "htod_gbs": round(n / ms / 1e6, 2), "htod_us": round(ms * 1e3, 2),
                    "dtoh_gbs": round(n / ms_d / 1e6, 2), "dtoh_us": round(ms_d * 1e3, 2), "wire_in": w,
                    "wire_out": wd, "ok": ok})
        del rings, dsts, outs, srcs, payload
        torch.cuda.empty_cache()
    return out


def c4(ctx, irregular):
    for proc, items in gen.C4_SCHEMAS.items():
        ctx.register_schema(proc, items)
    calls = gen.c4_calls(256 * MiB)
    ring = crk.Ring.device(1 << 29)
    cur, keep, reqs, outs, srcs = 0, [], [], [], []
    total = 0
    for c in calls:
        items = []
        for code, v in c.items:
            k = code & 0xFF
            if k in (crk.K_U32, crk.K_U64):
                items.append((code, v))
                continue
            t = torch.from_numpy(np.ascontiguousarray(v).view(np.uint8).copy()).to(dev)
            if k not in (crk.K_OPAQUE_VAR, crk.K_OPAQUE_FIX):
                t = t.view({4: torch.int32, 8: torch.int64}[crk.ELEM_SIZE[k]])
            items.append((code, t))
            keep.append(t)
        lens = None
        if irregular:
            L = ctx.call_logical_size(items)
            lens = gen.split_points(gen.frag_seed(c), L)
        cur += ctx.encode_call(c.xid, c.proc, items, ring, cur, frag_lens=lens)
        for a, (code, v) in enumerate(c.items):
            k = code & 0xFF
            if k in (crk.K_U32, crk.K_U64):
                continue
            nb = np.asarray(v).nbytes
            o = torch.empty(nb + 16, dtype=torch.uint8, device=dev)
            outs.append(o)
            srcs.append(items[a][1])
            reqs.append((c.xid, a, k, o.data_ptr(), len(v), None, None))
            total += nb
    torch.cuda.synchronize()
    idx = ctx.index(1, 1 << 16, 1 << 12)
    st = torch.zeros(len(reqs), dtype=torch.int32, device=dev)
    arr = (crk.ItemReq * len(reqs))(*[crk.ItemReq(a, b, k, 0, d, m, None, st.data_ptr() + 4 * i)
                                     for i, (a, b, k, d, m, _, _) in enumerate(reqs)])
    dreq = torch.frombuffer(bytearray(arr), dtype=torch.uint8).to(dev)

    def dec(_):
        idx.frame_scan([(ring, 0, cur)])
        crk._check(crk.lib().crk_xdr_decode_items_batch(ctx.h, idx.h, len(reqs), dreq.data_ptr(),
                                                         torch.cuda.current_stream().cuda_stream), "batch")

    ms = timed(dec, 10)
    ms_scan = timed_cold(lambda _: idx.frame_scan([(ring, 0, cur)]), 10)
    ok = bool((st == 0).all()) and all(torch.equal(o[:s.numel() * s.element_size()], s.view(torch.uint8).reshape(-1))
                                       for o, s in zip(outs, srcs))
    return {"records": len(calls), "items": len(reqs), "payload_bytes": total, "wire": cur, "ms": round(ms, 3),
            "scan_ms": round(ms_scan, 3), "frags": int(idx.ring_results(1)[0]["n_frags"]),
            "scan_stats": idx.scan_stats(),
            "decode_gbs": round(total / ms / 1e6, 1), "ok": ok}


def served(ctx, sizes_h2d, sizes_d2h, streams=1, reps=20):
    """Serve a batch of HtoD records (sizes_h2d) and DtoH records over `streams` rings; GB/s of payload."""
    total_h = sum(sizes_h2d)
    region = torch.zeros(total_h + sum(sizes_d2h) + 4096 * (len(sizes_h2d) + len(sizes_d2h)), dtype=torch.uint8,
                         device=dev)
    base = region.data_ptr()
    per = [[] for _ in range(streams)]
    off = 0
    srcs = []
    for i, n in enumerate(sizes_h2d):
        per[i % streams].append(("h", i, n, off))
        off += (n + 255) // 256 * 256
    for i, n in enumerate(sizes_d2h):
        per[i % streams].append(("d", i, n, off))
        region[off:off + n].copy_(torch.from_numpy(gen.random_bytes(7000 + i, n)))
        off += (n + 255) // 256 * 256
    rings, sends = [], []
    for s in range(streams):
        cap = next_pow2(sum(n + 64 + 4 * (n // 65536 + 2) for k, _, n, _ in per[s] if k == "h") + 64 * len(per[s]) + 4096)
        ring = crk.Ring.device(cap)
        cur = 0
        for k, i, n, o in per[s]:
            if k == "h":
                p = torch.from_numpy(gen.random_bytes(9000 + i, n)).to(dev)
                srcs.append((o, p))
                cur += ctx.encode_call(0x1000 * s + i + 1, gen.PROC_H2D,
                                       [(crk.K_U64, base + o), (crk.K_OPAQUE_VAR, p), (crk.K_U64, n)], ring, cur)
            else:
                cur += ctx.encode_call(0x800000 + 0x1000 * s + i, gen.PROC_D2H, [(crk.K_U64, base + o), (crk.K_U64, n)],
                                       ring, cur)
        rings.append((ring, 0, cur))
        sends.append(crk.Ring.device(next_pow2(sum(crk.wire_size_d2h(n, 0) for k, _, n, _ in per[s] if k == "d")
                                               + 64 * len(per[s]) + 4096)))
    idx = ctx.index(streams, 1 << 20, 1 << 14)
    ms = timed(lambda _: idx.serve(rings, sends, [0] * streams, base, region.numel()), reps)
    res = idx.ring_results(streams)
    ok = all(r["status"] == 0 and r["n_records"] == len(per[s]) for s, r in enumerate(res))
    # every destination; every ring's reply bytes (an HtoD reply carries a status, a DtoH one its data)
    F = ctx.cfg.frag_payload
    ok &= all(bool(torch.equal(region[o:o + p.numel()], p)) for o, p in srcs)
    ok &= all(r["reply_bytes"] == sum(crk.wire_size_d2h(0, 1, F) if k == "h" else crk.wire_size_d2h(n, 0, F)
                                      for k, _, n, _ in per[s]) for s, r in enumerate(res))
    ok &= all(bool(torch.equal(region[o:o + n].cpu(), torch.from_numpy(gen.random_bytes(7000 + i, n))))
              for s in range(streams) for k, i, n, o in per[s] if k == "d")  # DtoH sources untouched
    pay = total_h + sum(sizes_d2h)
    return {"ms": round(ms, 4), "payload_bytes": pay, "gbs": round(pay / ms / 1e6, 1), "ok": bool(ok)}


def striped(total, k, reps=20):
    """NEXT-1: one memcpy of `total` bytes striped over k rings (reading R22: k stripe CALLs, the offset-0 stripe
    carries the memcpy's reply), served as one crk_serve step; payload GB/s and the check."""
    ctx = Ctx()
    region = torch.zeros(total + 256, dtype=torch.uint8, device=dev)
    base = region.data_ptr()
    payload = torch.from_numpy(gen.random_bytes(0x51, total)).to(dev)
    per = total // k
    rings, sends = [], []
    for i in range(k):
        a, b = i * per, total if i == k - 1 else (i + 1) * per
        ring = crk.Ring.device(next_pow2(b - a + 4 * ((b - a) // 65536 + 2) + 128))
        w = ctx.encode_call(0x5100 + i, 3, [(crk.K_U64, base), (crk.K_OPAQUE_VAR, payload[a:b]), (crk.K_U64, b - a),
                                            (crk.K_U32, 0x51), (crk.K_U64, a), (crk.K_U64, total)], ring, 0)
        rings.append((ring, 0, w))
        sends.append(crk.Ring.device(4096))
    idx = ctx.index(k, 1 << 16, 1 << 10)
    ms = timed(lambda _: idx.serve(rings, sends, [0] * k, base, region.numel()), reps)
    res = idx.ring_results(k)
    ok = all(r["status"] == 0 for r in res) and res[0]["reply_bytes"] == 32 and sum(r["reply_bytes"] for r in res) == 32
    ok &= bool(torch.equal(region[:total], payload))
    return {"ms": round(ms, 4), "stripes": k, "payload_bytes": total, "gbs": round(total / ms / 1e6, 1), "ok": bool(ok),
            "scan_stats": idx.scan_stats()}


def profile(streams, region_bytes, reps=10):
    """A gen workload profile (NEXT-2) served by crk_serve: payload GB/s and the per-ring check."""
    from paper_conf_sc_eilingkkflm23_b200 import workload
    ctx = Ctx()
    ep = workload.endpoint(ctx, 0, dev, streams, region_bytes)
    idx = ctx.index(len(streams), 1 << 16, 1 << 12)
    ms = timed(lambda _: workload.serve_step(idx, ep), reps)
    chk = workload.check_results(idx, ep)
    return {"ms": round(ms, 4), "payload_bytes": ep.payload, "records": ep.n_records, "streams": len(streams),
            "gbs": round(ep.payload / ms / 1e6, 1), "ok": chk["ok"], "scan_stats": idx.scan_stats()}


def main():
    build.build()
    only = [x for x in os.environ.get("SUITE_ONLY", "").split(",") if x]
    runs = {
        "C1": lambda: c1(Ctx()),
        "C1_serve_one_record": lambda: serve_latency(Ctx()),
        "C1_serve_one_record_general": lambda: serve_latency(crk.Context(0, **{**CTX_KW, "lean_steps": 0})),
        "C2_matrixMul": lambda: c2(Ctx()),
        "NEXT3_server": lambda: server_latency(Ctx()),
        "NEXT3_server_general": lambda: server_latency(crk.Context(0, **{**CTX_KW, "lean_steps": 0}), reps=500),
        "C3_sweep": lambda: c3(Ctx()),
        "C4_typed_regular": lambda: c4(Ctx(), False),
        "C4_typed_irregular": lambda: c4(Ctx(), True),
        "NEXT1_striped_1GiB_16_rings": lambda: striped(GiB, 16),
        "NEXT1_striped_1GiB_4_rings": lambda: striped(GiB, 4),
        "NEXT1_single_1GiB_1_ring": lambda: served(Ctx(), [GiB], [], streams=1),
        "NEXT1_16_separate_64MiB_calls": lambda: served(Ctx(), [64 * MiB] * 16, [], streams=16),
        "NEXT2_cusolver_100_iters": lambda: profile(*gen.cusolver_endpoint(iterations=100)),
        "NEXT2_cusolver_100_iters_4_streams": lambda: profile(*gen.cusolver_endpoint(iterations=100, n_streams=4)),
        "NEXT2_histogram": lambda: profile(*gen.histogram_endpoint()),
    }
    out = {}
    t0 = time.time()
    for name, fn in runs.items():
        if not only or any(name.startswith(o) for o in only):
            out[name] = fn()
    out["wall_s"] = round(time.time() - t0, 1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
