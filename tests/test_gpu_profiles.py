"""GPU parity of the NEXT-2 workload profiles: the memcpy traffic of the paper's
cuSolverDn_LinearSolver (900 x 900 LU; 6.07 GiB in 1000 iterations) and histogram
(64 MiB) applications, drawn by gen.cusolver_endpoint / gen.histogram_endpoint, encoded on the
GPU by workload.endpoint, served by crk_serve, and compared byte for byte with the oracle's or_serve on its own
encoding of the same draws (tests/c5_oracle.py): the whole region, every send ring, every per-record status."""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import crk, gen, workload
from tests.c5_oracle import oracle_endpoint_of

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("needs a GPU", allow_module_level=True)


def serve_and_compare(streams, region_bytes, **ctx_kw):
    dev = torch.device("cuda:0")
    ctx = crk.Context(0, **ctx_kw)
    ep = workload.endpoint(ctx, 0, dev, streams, region_bytes)
    idx = ctx.index(len(streams), 1 << 16, 1 << 12)
    ep.region[:region_bytes].fill_(0)  # HtoD destinations start zeroed; DtoH sources are re-placed below
    oe = oracle_endpoint_of(streams, region_bytes, ep.base)
    ep.region.copy_(torch.from_numpy(oe.region).to(dev))
    for (ring, h, t), w in zip(ep.rings, oe.wires):  # the GPU encoder's rings are the oracle's encoding
        assert h == 0 and torch.equal(ring.tensor()[:t].cpu(), torch.from_numpy(w))
    idx.serve(ep.rings, ep.sends, ep.offs, ep.base, ep.region.numel())
    torch.cuda.synchronize()
    want = O.serve([(oe.ring_array(i, r.cap), 0, len(w)) for i, ((r, _, _), w) in enumerate(zip(ep.rings, oe.wires))],
                   oe.cfg, oe.region, ep.base, [s.cap for s in ep.sends], ep.offs,
                   max_frags_per_ring=(1 << 16) // len(streams), max_records_per_ring=(1 << 12) // len(streams))
    assert all(s == O.OK for s in want["scan_status"])
    assert all(r["status"] == O.OK for r in want["records"])
    T = idx.tables(len(streams))
    assert [r["status"] for r in want["records"]] == list(T["parsed"]["serve_status"])
    assert torch.equal(ep.region, torch.from_numpy(oe.region).to(dev))
    for r, send in enumerate(ep.sends):
        n = want["reply_bytes"][r]
        assert T["rings"][r]["reply_bytes"] == n
        assert torch.equal(send.tensor()[:n].cpu(), torch.from_numpy(want["send"][r][:n]))
    return idx


@pytest.mark.parametrize("n_streams", [1, 4])
def test_cusolver_profile_matches_oracle(n_streams):
    streams, rb = gen.cusolver_endpoint(iterations=12, n_streams=n_streams)
    serve_and_compare(streams, rb)


def test_histogram_profile_matches_oracle():
    streams, rb = gen.histogram_endpoint()
    idx = serve_and_compare(streams, rb)
    assert idx.scan_stats()["chunked"] == 1  # the 64 MiB record goes through the chunked scan
