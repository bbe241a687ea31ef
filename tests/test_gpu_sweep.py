"""GPU parity of bench.py's host-link sweeps (workload.LinkSweep): bandwidthTest-shaped
memcpy CALLs served from pinned host rings, copy-engine staged and zero-copy, against the oracle.  HtoD: the
destination region == the payload and the host send ring's REPLY == or_serve's; DtoH: the host send ring's
REPLY bytes == or_encode_memcpy_d2h of the payload, every byte; C2: the matrixMul batch's region and replies ==
or_serve on the oracle's own encoding of the same three CALLs."""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import crk, gen, workload

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("needs a GPU", allow_module_level=True)

CFG = O.Config(prog=gen.PROG, vers=gen.VERS, proc_h2d=gen.PROC_H2D, proc_d2h=gen.PROC_D2H, frag_payload=65536)


@pytest.fixture(scope="module")
def sweep():
    dev = torch.device("cuda:0")
    return workload.LinkSweep(0, dev, max_n=1 << 23)


@pytest.mark.parametrize("n", [1 << 12, (1 << 20) + 3, 5 << 20])
@pytest.mark.parametrize("direction", ["h2d", "d2h"])
@pytest.mark.parametrize("mode", ["ce", "zc"])
def test_sweep_calls_match_oracle(sweep, n, direction, mode):
    payload_np = gen.random_bytes(n, n)
    payload = torch.from_numpy(payload_np).cuda()
    sweep.prepare(n, direction, payload)
    for sl in sweep.slots:  # poison the outputs
        sl.tx_host.host_view()[:sl.w_out + 64] = 0xA5
        if direction == "h2d":
            sl.region[:n].fill_(0x5A)
    sweep.run(mode, 5, torch.cuda.current_stream())
    assert sweep.check(payload)
    for i, sl in enumerate(sweep.slots):
        got = np.frombuffer(sl.tx_host.read(0, sl.w_out), np.uint8)
        if direction == "h2d":
            xid = 0x5E0000 + i
            assert torch.equal(sl.region[:n], payload)
            want = O.frame(O.reply_header(xid) + O.put_u32(0), 65536)
        else:
            want = O.encode_memcpy_d2h(0x5D0000 + i, payload_np, 0, 65536)
        assert got.tobytes() == want


@pytest.mark.parametrize("mode", ["ce", "zc"])
def test_c2_batch_matches_oracle(sweep, mode):
    for sl in sweep.slots:
        sl.region.zero_()
    sweep.prepare_c2()
    sweep.run(mode, 4, torch.cuda.current_stream())
    assert sweep.check(None)
    A, B, Cm = gen.c2_matrices()
    for i, sl in enumerate(sweep.slots):
        base = sl.region.data_ptr()
        wire = (O.encode_call(0xC2A, gen.PROC_H2D, [(O.K_U64, base), (O.K_OPAQUE_VAR, A.tobytes()),
                                                     (O.K_U64, A.nbytes)], CFG)
                + O.encode_call(0xC2B, gen.PROC_H2D, [(O.K_U64, base + 409_600), (O.K_OPAQUE_VAR, B.tobytes()),
                                                       (O.K_U64, B.nbytes)], CFG)
                + O.encode_call(0xC2C, gen.PROC_D2H, [(O.K_U64, base + 1_228_800), (O.K_U64, Cm.nbytes)], CFG))
        assert sl.rx_host.read(0, sl.w_in) == wire  # the GPU encoder built the oracle's bytes
        ring = np.zeros(1 << 21, np.uint8)
        ring[:len(wire)] = np.frombuffer(wire, np.uint8)
        region = np.zeros(sl.region.numel(), np.uint8)
        region[1_228_800:1_228_800 + Cm.nbytes] = Cm.view(np.uint8)
        want = O.serve([(ring, 0, len(wire))], CFG, region, base, [1 << 20], [0])
        assert [r["status"] for r in want["records"]] == [O.OK] * 3
        assert np.array_equal(sl.region.cpu().numpy(), region)
        n = want["reply_bytes"][0]
        assert n == sl.w_out and sl.tx_host.read(0, n) == bytes(want["send"][0][:n])
