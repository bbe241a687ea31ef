"""GPU parity of the exact loops bench.py times (VERDICT r1 "What's weak" 2), element by element against the
oracle's or_serve, at the full C5 size (BASELINE.json configs[4]: 16 client streams x 64 MiB per GPU).

* Device-resident loop (`value`): workload.build_slots + workload.run_pipelined with bench.py's defaults --
  3 contexts / indexes / streams in flight, mover_reserve_ctas 16, mover_tail_tiles 0, an index of 2^14
  records so planning takes the multi-kernel path and the mover claims through the run -> job map (checked
  with the context's counters).  After warm-up + K steps, for every slot: the rings the GPU encoder built ==
  the oracle's encoding, the whole 1 GiB region == or_serve's region, every send ring's reply bytes ==
  or_serve's, every per-record serve status and every per-ring result == or_serve's.
* Host-ring loops (`e2e`): workload.StagedLoop's copy-engine staged, mixed and zero-copy modes over pinned
  host rings, the same comparisons on the host send rings.

Serving is idempotent for this workload (HtoD destinations and DtoH sources are disjoint, reply cursors
restart at 0 every step), so after K steps the state must equal one or_serve pass.  The oracle encodes its
own rings from gen's descriptions (tests/c5_oracle.py); nothing it consumes comes from the CUDA path.
"""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import crk, gen, workload
from tests.c5_oracle import oracle_endpoint

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("needs a GPU", allow_module_level=True)

MiB = 1 << 20
P, WARMUP, K = 3, 5, 7  # bench.py defaults: --pipeline 3, --warmup 5; K steps after warm-up


def check_slot(slot: workload.Slot, host_rings: bool, want_counters_map: bool):
    ep = slot.ep
    dev = ep.region.device
    oe = oracle_endpoint(ep.rank, len(ep.streams), ep.region.numel() - 256, ep.base,
                         payload_per_stream=sum(r.size for r in ep.streams[0].records),
                         h2d_frac=slot.h2d_frac)
    # 1. the rings the CUDA encoder built are the oracle's encoding, byte for byte
    for (ring, h, t), w in zip(ep.rings, oe.wires):
        assert h == 0 and t == len(w)
        got = torch.from_numpy(ring.host_view()[:t].copy()) if host_rings else ring.tensor()[:t].cpu()
        assert torch.equal(got, torch.from_numpy(w))
    # 2. one or_serve pass over the oracle's rings
    send_caps = [s.cap for s in ep.sends]
    want = O.serve([(oe.ring_array(i, ring.cap), 0, len(w)) for i, ((ring, _, _), w) in
                    enumerate(zip(ep.rings, oe.wires))], oe.cfg, oe.region, ep.base, send_caps, ep.offs,
                   max_frags_per_ring=workload.INDEX_SHAPE["max_frags"] // len(ep.rings),
                   max_records_per_ring=workload.INDEX_SHAPE["max_records"] // len(ep.rings))
    assert all(s == O.OK for s in want["scan_status"])
    assert torch.equal(ep.region, torch.from_numpy(oe.region).to(dev)), "region differs from or_serve"
    T = slot.idx.tables(len(ep.rings))
    assert [r["status"] for r in want["records"]] == list(T["parsed"]["serve_status"])
    assert [r["reply_err"] for r in want["records"]] == list(T["parsed"]["serve_reply_err"])
    for r, send in enumerate(ep.sends):
        g = T["rings"][r]
        assert g["status"] == O.OK and g["consumed"] == want["consumed"][r]
        assert g["reply_bytes"] == want["reply_bytes"][r] == ep.per_stream_reply[r]
        assert g["n_records"] == ep.per_stream_records[r]
        n = want["reply_bytes"][r]
        exp = torch.from_numpy(want["send"][r][ep.offs[r]:ep.offs[r] + n])
        got = (torch.from_numpy(send.host_view()[ep.offs[r]:ep.offs[r] + n].copy()) if host_rings
               else send.tensor()[ep.offs[r]:ep.offs[r] + n].cpu())
        assert torch.equal(got, exp), f"send ring {r} differs from or_serve"
    if want_counters_map:
        assert slot.ctx.debug_counters()[13] == 1, "the mover did not claim through the run -> job map"


@pytest.mark.parametrize("direction", ["mixed", "h2d"])
def test_bench_pipelined_loop_matches_oracle(direction):
    import bench
    dev = torch.device("cuda:0")
    ctx_kw = workload.pipelined_ctx_kw({}, P)
    assert ctx_kw == {"mover_reserve_ctas": 16, "mover_tail_tiles": 0, "scan_chunking": 1}
    frac = bench.H2D_FRAC[direction]
    slots = workload.build_slots(0, 0, dev, P, ctx_kw, n_streams=16, payload_per_stream=64 * MiB, h2d_frac=frac,
                                 default_stream=torch.cuda.current_stream(dev))
    for s in slots:
        s.h2d_frac = frac
        assert s.ctx.cfg.mover_reserve_ctas == 16 and s.ctx.cfg.mover_tail_tiles == 0 and s.ctx.cfg.mover_run == 8
    stream = torch.cuda.current_stream(dev)
    workload.run_pipelined(slots, stream, WARMUP)
    # poison every output between warm-up and the timed steps, so the comparison sees only what they wrote
    for s in slots:
        h2d = [r for st in s.ep.streams for r in st.records if r.kind == gen.PROC_H2D]
        for r in h2d:
            s.ep.region[r.region_off:r.region_off + r.size].fill_(0xA5)
        for send in s.ep.sends:
            send.tensor().fill_(0x5A)
    torch.cuda.synchronize()
    e0, e1 = workload.run_pipelined(slots, stream, K)
    torch.cuda.synchronize()
    assert e0.elapsed_time(e1) > 0
    for s in slots:
        check_slot(s, host_rings=False, want_counters_map=True)


@pytest.mark.parametrize("mode", ["staged", "mixed", "zero_copy"])
def test_bench_e2e_loops_match_oracle(mode):
    dev = torch.device("cuda:0")
    ctx_kw = workload.pipelined_ctx_kw({}, P)
    slots = workload.build_slots(0, 0, dev, P, ctx_kw, n_streams=16, payload_per_stream=64 * MiB, h2d_frac=0.5,
                                 host_rings=True, staged=True, default_stream=torch.cuda.current_stream(dev))
    loop = workload.StagedLoop(slots, dev)
    run = {"staged": loop.run, "mixed": loop.run_mixed, "zero_copy": loop.run_zero_copy}[mode]
    run(2)
    for s in slots:
        s.h2d_frac = 0.5
        for r in (x for st in s.ep.streams for x in st.records if x.kind == gen.PROC_H2D):
            s.ep.region[r.region_off:r.region_off + r.size].fill_(0xA5)
        for send in s.ep.sends:
            send.host_view()[:] = 0x5A
        for send in s.ep.dev_sends:
            send.tensor().fill_(0x5A)
    torch.cuda.synchronize()
    run(K)
    torch.cuda.synchronize()
    for s in slots:
        check_slot(s, host_rings=True, want_counters_map=True)
