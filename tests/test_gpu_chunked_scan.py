"""GPU parity of the chunked multi-CTA scan (k_mscan.cu; DESIGN.md §8 K1) against the oracle's or_frame_scan
(RFC 5531 §11), field by field, on windows long enough to be cut into chunks.

The chunked scan guesses each chunk's entry from its landing zone and keeps a guess only when the previous
chunk's true chain exits exactly there; when no guess fits it falls back to the one-CTA scan.  Every case
below is compared with the oracle whichever way it went; the cases the design is for (greedy 64 KiB framing,
C4-ii irregular framing, mixed HtoD / DtoH streams, host rings) must also resolve without a fallback
(`Index.scan_stats`), and the cases it cannot guess (fragments > 64 KiB, long runs of tiny fragments,
payloads of zeros) must fall back and still match."""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import gen
from tests.gpu_util import compare_parse, compare_scan, ctx_for, d2h_call, h2d_call, make_ring, ocfg, ring_np

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("needs a GPU", allow_module_level=True)

MiB = 1 << 20


def place(ring, wire: bytes, at: int) -> int:
    ring.write(at, wire)
    return at + len(wire)


def c5_like(seed: int, total: int, cfg, F=65536, lo=4096, hi=4 * MiB, payload=None):
    """HtoD / DtoH memcpy CALLs (50/50), sizes log-uniform, until `total` wire bytes."""
    g = gen.rng(seed)
    wires, n = [], 0
    i = 0
    while n < total:
        size = gen.log_uniform_int(g, lo, hi)
        if g.random() < 0.5:
            d = payload(size, i) if payload else gen.random_bytes(seed * 1000 + i, size)
            w = O.encode_call(*h2d_call(0x100000 + i, d), cfg, F=F)
        else:
            w = O.encode_call(*d2h_call(0x100000 + i, 0x7F0000000000 + i * 64, size), cfg, F=F)
        wires.append(w)
        n += len(w)
        i += 1
    return wires


def irregular(seed: int, total: int, cfg, hi=65536):
    """C4-ii framing: fragment lengths uniform in [1, hi] (gen.split_points)."""
    g = gen.rng(seed)
    wires, n, i = [], 0, 0
    while n < total:
        d = gen.random_bytes(seed * 7 + i, gen.log_uniform_int(g, 1, 2 * MiB))
        L = O.call_header(0x200000 + i, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0) + \
            O.put_opaque_var(d.tobytes()) + O.put_u64(len(d))
        w = O.frame_lens(L, gen.split_points(seed * 131 + i, len(L), 1, hi))
        wires.append(w)
        n += len(w)
        i += 1
    return wires


def run_scan(wires, head=0, cap=1 << 24, host=False, fpr=1 << 16, rpr=1 << 12, cut=None, user=None, mrb=1 << 32,
             parse=True, **kw):
    cfg = ocfg(user=user)
    ctx = ctx_for(cfg, max_record_bytes=mrb, **kw)
    ring = make_ring(cap, host)
    tail = head
    for w in wires:
        tail = place(ring, w, tail)
    if cut is not None:
        tail = head + cut
    idx = ctx.index(1, fpr, rpr)
    idx.frame_scan([(ring, head, tail)])
    T = idx.tables()
    rb = ring_np(ring)
    s = compare_scan(T, 0, rb, head, tail, fpr, rpr, max_record_bytes=mrb)
    if parse:
        compare_parse(T, 0, rb, s, cfg)
    return s, idx.scan_stats(), tail - head


@pytest.mark.parametrize("host", [False, True])
@pytest.mark.parametrize("head", [0, (1 << 24) - 100003])
def test_c5_like_stream_resolves_chunked(host, head):
    wires = c5_like(1, 12 * MiB, ocfg())
    s, st, w = run_scan(wires, head=head, host=host)
    assert s.status == O.OK and len(s.recs) == len(wires)
    assert w >= 2 * 256 * 1024 and st == {"chunked": 1, "fallback": 0}, st


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_irregular_framing_resolves_chunked(seed):
    wires = irregular(seed, 10 * MiB, ocfg())
    s, st, _ = run_scan(wires, head=seed * 999)
    assert s.status == O.OK and len(s.recs) == len(wires)
    assert st == {"chunked": 1, "fallback": 0}, st


def test_truncations_across_chunks():
    """Windows ending inside a header, inside fragment data, at an exact record boundary, one byte short."""
    wires = c5_like(4, 3 * MiB, ocfg(), hi=MiB)
    full = sum(len(w) for w in wires)
    ends = np.cumsum([len(w) for w in wires])
    g = gen.rng(9)
    cuts = sorted(set([full, full - 1, int(ends[len(ends) // 2]), int(ends[len(ends) // 2]) + 2] +
                      [int(x) for x in g.integers(600 * 1024, full, 6)]))
    cfg = ocfg()
    ctx = ctx_for(cfg)
    ring = make_ring(1 << 23)
    tail = 0
    for w in wires:
        tail = place(ring, w, tail)
    rb = ring_np(ring)
    idx = ctx.index(1, 1 << 16, 1 << 12)
    for c in cuts:
        idx.frame_scan([(ring, 0, c)])
        s = compare_scan(idx.tables(), 0, rb, 0, c, 1 << 16, 1 << 12)
        assert s.status == (O.OK if c in (full, int(ends[len(ends) // 2])) else O.INCOMPLETE)
    assert idx.scan_stats()["fallback"] == 0


def test_frag_limit_and_capacity_stops():
    wires = c5_like(5, 6 * MiB, ocfg(), hi=2 * MiB)
    sizes = sorted(len(w) for w in wires)
    # E_FRAG: the first record longer than max_record_bytes, wherever it falls among the chunks
    s, st, _ = run_scan(wires, mrb=sizes[len(sizes) // 2], parse=False)
    assert s.status == O.E_FRAG
    # fragment capacity runs out mid-window (INCOMPLETE with records kept) / before any record (E_CAPACITY)
    s, _, _ = run_scan(wires, fpr=40, parse=False)
    assert s.status in (O.INCOMPLETE, O.E_CAPACITY)
    s, _, _ = run_scan(wires, rpr=3, parse=False)
    assert s.status == O.INCOMPLETE and len(s.recs) == 3


def test_zero_length_fragments_and_mixed_framings():
    cfg = ocfg(user={33: [O.K_U32]})
    g = gen.rng(12)
    wires = []
    for i in range(60):
        d = gen.random_bytes(i + 50, int(g.integers(0, 300000)))
        L = O.call_header(i, gen.PROG, gen.VERS, gen.PROC_H2D) + O.put_u64(0) + O.put_opaque_var(d.tobytes()) + \
            O.put_u64(len(d))
        lens = gen.split_points(i, len(L), 1, int(g.choice([4000, 65536])))
        for _ in range(int(g.integers(0, 3))):
            lens.insert(int(g.integers(0, len(lens) + 1)), 0)  # reading R1
        if g.random() < 0.3:
            lens.append(0)  # reading R2
        wires.append(O.frame_lens(L, lens))
        wires.append(O.encode_call(9000 + i, 33, [(O.K_U32, i)], cfg))
    s, st, _ = run_scan(wires, user={33: [O.K_U32]})
    assert s.status == O.OK and len(s.recs) == 120


@pytest.mark.parametrize("case", ["big_fragments", "tiny_fragments", "zero_payload", "small_int_payload"])
def test_unguessable_framings_fall_back_and_match(case):
    cfg = ocfg()
    if case == "big_fragments":  # fragments of 1 MiB: a chunk's entry lies beyond its landing zone
        wires = c5_like(6, 6 * MiB, cfg, F=1 << 20, lo=1 << 20)
    elif case == "tiny_fragments":  # 200-byte fragments: more headers per chunk than a log holds
        wires = c5_like(7, 3 * MiB, cfg, F=200, lo=256 * 1024, hi=MiB)
    elif case == "zero_payload":  # every zone position parses as a zero-length header
        wires = c5_like(8, 6 * MiB, cfg, payload=lambda n, i: np.zeros(n, np.uint8))
    else:  # big-endian small integers: many plausible headers in every zone
        wires = c5_like(9, 6 * MiB, cfg, payload=lambda n, i: np.frombuffer(
            (np.arange((n + 3) // 4, dtype=np.uint32) % 5000).astype(">u4").tobytes()[:n], np.uint8))
    s, st, _ = run_scan(wires, fpr=1 << 18)
    assert s.status == O.OK and len(s.recs) == len(wires)
    assert st["chunked"] + st["fallback"] == 1
    if case in ("big_fragments", "tiny_fragments"):
        assert st["fallback"] == 1


def test_many_rings_long_and_short_in_one_launch():
    cfg = ocfg()
    ctx = ctx_for(cfg)
    rings, wins = [], []
    for r in range(6):
        wires = c5_like(20 + r, [100_000, 5 * MiB, 200, 3 * MiB, 0, 9 * MiB][r], cfg) if r != 4 else []
        ring = make_ring(1 << 24)
        head = r * 4093
        tail = head
        for w in wires:
            tail = place(ring, w, tail)
        rings.append(ring)
        wins.append((head, tail))
    idx = ctx.index(6, 6 << 14, 6 << 10)
    idx.frame_scan([(ring, h, t) for ring, (h, t) in zip(rings, wins)])
    T = idx.tables(6)
    for r, (ring, (h, t)) in enumerate(zip(rings, wins)):
        rb = ring_np(ring)
        s = compare_scan(T, r, rb, h, t, 1 << 14, 1 << 10)
        compare_parse(T, r, rb, s, cfg)
    st = idx.scan_stats()
    assert st["fallback"] == 0 and st["chunked"] >= 2


def test_chunking_off_matches_too():
    wires = irregular(4, 4 * MiB, ocfg())
    s, st, _ = run_scan(wires, scan_chunking=1)
    assert s.status == O.OK and st == {"chunked": 0, "fallback": 0}


def test_serve_through_chunked_scan_matches_oracle():
    """The whole server step (scan, parse, plan, movers) over long rings, against or_serve."""
    cfg = ocfg(F=65536)
    ctx = ctx_for(cfg)
    streams, region_bytes = gen.c5_endpoint(3, n_streams=3, payload_per_stream=12 * MiB, h2d_budget=11 * MiB,
                                            misalign=True)
    region = torch.zeros(region_bytes + 64, dtype=torch.uint8, device="cuda")
    base = region.data_ptr()
    host_region = np.zeros(region_bytes + 64, np.uint8)
    rings, sends, offs = [], [], []
    for s in streams:
        ring = make_ring(1 << 24)
        cur = 77 * s.stream
        for r in s.records:
            d = gen.random_bytes(r.seed & 0xFFFFFFFF, r.size)
            if r.kind == gen.PROC_D2H:
                host_region[r.region_off:r.region_off + r.size] = d
                c = d2h_call(r.xid, base + r.region_off, r.size)
            else:
                c = h2d_call(r.xid, d, base + r.region_off)
            cur = place(ring, O.encode_call(*c, cfg), cur)
        rings.append((ring, 77 * s.stream, cur))
        sends.append(make_ring(1 << 24))
        offs.append(5 * s.stream)
    region.copy_(torch.from_numpy(host_region))
    idx = ctx.index(3, 3 << 13, 3 << 10)
    idx.serve(rings, sends, offs, base, region_bytes + 64)
    torch.cuda.synchronize()
    st = idx.scan_stats()  # the DtoH-heavy ring's window (60-byte CALLs) can be short: one CTA
    assert st["fallback"] == 0 and st["chunked"] >= 2, st
    T = idx.tables(3)
    want = O.serve([(ring_np(r), h, t) for r, h, t in rings], cfg, host_region, base, [1 << 24] * 3, offs,
                   max_frags_per_ring=1 << 13, max_records_per_ring=1 << 10)
    assert np.array_equal(region.cpu().numpy(), host_region)
    assert [r["status"] for r in want["records"]] == list(T["parsed"]["serve_status"])
    for r in range(3):
        n = want["reply_bytes"][r]
        assert T["rings"][r]["reply_bytes"] == n and T["rings"][r]["consumed"] == want["consumed"][r]
        assert sends[r].read(offs[r], n) == bytes(want["send"][r][offs[r]:offs[r] + n])


@pytest.mark.parametrize("case", ["one_call_24MiB", "irregular_capped", "capacity_stop"])
def test_capped_small_index_takes_the_fused_front_end(case):
    """A small index (<= fused_front_max_records records, <= fused_front_max_frags fragments in all) scans a
    window past fused_front_max_window in the fused single-CTA front end -- its capacity bounds the header
    walk -- and still equals or_frame_scan / or_parse_call; the same window over a larger index is chunked."""
    cfg = ocfg()
    if case == "one_call_24MiB":  # one C3-shaped memcpy CALL: 385 headers
        d = gen.random_bytes(77, 24 * MiB)
        wires, fpr, rpr = [O.encode_call(*h2d_call(0xC3, d), cfg)], 400, 4
    elif case == "irregular_capped":  # C4-ii framing, fragments uniform in [1, 64 KiB]: every hop a new length
        wires, fpr, rpr = irregular(31, 40 * MiB, cfg), 2048, 128
    else:  # more records than the index holds: the one CTA stops at the record capacity
        wires, fpr, rpr = c5_like(32, 8 * MiB, cfg, hi=256 * 1024), 2048, 16
    s, st, w = run_scan(wires, head=12345, cap=1 << 26, fpr=fpr, rpr=rpr)
    assert w > (1 << 20) and st == {"chunked": 0, "fallback": 0}, st  # past the window limit, yet fused
    if case == "one_call_24MiB":
        assert s.status == O.OK and len(s.recs) == 1
    if case == "capacity_stop":
        assert s.status == O.INCOMPLETE and len(s.recs) == rpr
    s2, st2, _ = run_scan(wires, head=12345, cap=1 << 26, fpr=fpr, rpr=rpr, fused_front_max_frags=0)
    assert st2["chunked"] + st2["fallback"] == 1 and s2.status == s.status and len(s2.recs) == len(s.recs)
