"""Builds the benchmark workloads on the GPU with the library's own encoder (no oracle involved).

C5 endpoint (BASELINE.json configs[4], one per GPU): 16 client streams, each a ring of memcpy CALL
records (sizes log-uniform 4 KiB-16 MiB, 50/50 HtoD/DtoH, 64 MiB of payload per stream, 1 GiB per GPU),
framed with F = 64 KiB fragments.  The HtoD payloads and the DtoH source bytes come
from gen's seeded streams; the CALL records are encoded into the rings by crk_rpc_encode_call (the
client side of the same codec).  Ring filling is setup, outside every timed region.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np
import torch

from . import crk, gen

MiB = 1 << 20


def next_pow2(x: int) -> int:
    return 1 << max(8, (max(1, x) - 1).bit_length())


@dataclass
class Endpoint:
    ctx: crk.Context
    rank: int
    streams: list
    region: torch.Tensor
    rings: list = field(default_factory=list)       # (Ring, head, tail)
    sends: list = field(default_factory=list)       # Ring
    offs: list = field(default_factory=list)
    h2d_payload: int = 0
    d2h_payload: int = 0
    wire_in: int = 0
    reply_wire: int = 0
    n_records: int = 0
    per_stream_reply: list = field(default_factory=list)
    per_stream_records: list = field(default_factory=list)
    dev_rings: list = field(default_factory=list)   # staged mode: device copies of the host rings
    dev_sends: list = field(default_factory=list)

    @property
    def base(self) -> int:
        return self.region.data_ptr()

    @property
    def payload(self) -> int:
        return self.h2d_payload + self.d2h_payload


def c5_endpoint(ctx: crk.Context, rank: int, device: torch.device, n_streams: int = 16,
                payload_per_stream: int = 64 * MiB, host_rings: bool = False, misalign: bool = False,
                staged: bool = False, h2d_frac: float = 0.5) -> Endpoint:
    """h2d_frac: share of HtoD calls (0.5 = the mixed 50/50 stream; 1.0 / 0.0 = HtoD-only / DtoH-only,
    SURVEY.md §8(d) C5's three directions)."""
    budget = payload_per_stream if h2d_frac >= 1.0 else payload_per_stream - payload_per_stream // 16
    streams, region_bytes = gen.c5_endpoint(rank, n_streams=n_streams, payload_per_stream=payload_per_stream,
                                            h2d_budget=budget, misalign=misalign, h2d_frac=h2d_frac)
    return endpoint(ctx, rank, device, streams, region_bytes, host_rings=host_rings, staged=staged)


def endpoint(ctx: crk.Context, rank: int, device: torch.device, streams: list, region_bytes: int,
             host_rings: bool = False, staged: bool = False) -> Endpoint:
    """An endpoint serving gen's memcpy streams (C5, or the NEXT-2 profiles): one ring per stream holding its
    CALLs (encoded on the GPU), one send ring per stream, one device region for every HtoD destination and
    DtoH source."""
    region = torch.zeros(region_bytes + 256, dtype=torch.uint8, device=device)
    ep = Endpoint(ctx, rank, streams, region)
    F = ctx.cfg.frag_payload
    for s in streams:
        # wire size of every record from the library's closed forms, to size the rings
        h2d = [r for r in s.records if r.kind == gen.PROC_H2D]
        d2h = [r for r in s.records if r.kind == gen.PROC_D2H]
        stage_cap = max([r.size for r in h2d] + [1])
        stage = torch.empty(stage_cap + 16, dtype=torch.uint8, device=device)
        ring_dev = crk.Ring.device(next_pow2(sum(r.size + 64 + 4 * (r.size // F + 2) for r in h2d) + 64 * len(d2h)
                                             + 4096), device)
        cur = 0
        for r in s.records:
            data = torch.from_numpy(gen.random_bytes(r.seed & 0xFFFFFFFF, r.size)).to(device)
            if r.kind == gen.PROC_H2D:
                stage[:r.size].copy_(data)
                items = [(crk.K_U64, ep.base + r.region_off), (crk.K_OPAQUE_VAR, stage[:r.size]),
                         (crk.K_U64, r.size)]
                ep.h2d_payload += r.size
            else:
                ep.region[r.region_off:r.region_off + r.size].copy_(data)
                items = [(crk.K_U64, ep.base + r.region_off), (crk.K_U64, r.size)]
                ep.d2h_payload += r.size
            cur += ctx.encode_call(r.xid, r.kind, items, ring_dev, cur)
            torch.cuda.synchronize(device)
        reply = sum(crk.wire_size_d2h(r.size, 0, F) for r in d2h) + sum(crk.wire_size_d2h(0, 1, F) for _ in h2d)
        if host_rings:
            ring = crk.Ring.host(ring_dev.cap)
            torch.cuda.synchronize(device)
            host = torch.from_numpy(ring.host_view())
            host[:cur].copy_(ring_dev.tensor()[:cur].cpu())
            send = crk.Ring.host(next_pow2(reply + 4096))
            if staged:  # device rings the copy engine stages into / out of (crk_ring_copy)
                ring_dev.tensor().zero_()
                ep.dev_rings.append(ring_dev)
                ep.dev_sends.append(crk.Ring.device(send.cap, device))
            else:
                del ring_dev
        else:
            ring = ring_dev
            send = crk.Ring.device(next_pow2(reply + 4096), device)
        ep.rings.append((ring, 0, cur))
        ep.sends.append(send)
        ep.offs.append(0)
        ep.wire_in += cur
        ep.reply_wire += reply
        ep.n_records += len(s.records)
        ep.per_stream_reply.append(reply)
        ep.per_stream_records.append(len(s.records))
        del stage
    torch.cuda.synchronize(device)
    return ep


@dataclass
class Slot:
    """One in-flight batch of a pipelined server loop: its own context (scratch), index, stream and
    batch buffers, so consecutive batches overlap without sharing state."""
    ctx: crk.Context
    idx: crk.Index
    ep: Endpoint
    stream: torch.cuda.Stream
    res: "crk.PinnedResults | None" = None


# Settings of the pipelined server loop (bench.py's timed configuration): with batches in flight the mover
# leaves 16 CTA slots free, so the next batch's front-end kernels and the start of its mover overlap this one,
# and claims whole runs to the end (its CTAs retire staggered, handing SMs over gradually).  The front end
# uses the one-CTA-per-ring scan there: it runs inside those 16 free slots while the previous batch's mover
# streams, whereas the chunked scan needs ~2 CTAs on every SM and would wait for the mover to leave
# (measured: 0.374 vs 0.335 ms per C5 step).  A batch served alone (latency) takes the chunked scan.
PIPELINE_CTX = {"mover_reserve_ctas": 16, "mover_tail_tiles": 0, "scan_chunking": 1}
INDEX_SHAPE = dict(max_frags=1 << 20, max_records=1 << 14)  # per endpoint (16 rings): > kSmallServe records


def pipelined_ctx_kw(ctx_kw: dict, pipeline: int) -> dict:
    kw = dict(ctx_kw)
    if pipeline > 1:
        for k, v in PIPELINE_CTX.items():
            kw.setdefault(k, v)
    return kw


def build_slots(device_index: int, rank: int, device: torch.device, pipeline: int, ctx_kw: dict,
                n_streams: int = 16, payload_per_stream: int = 64 * MiB, h2d_frac: float = 0.5,
                host_rings: bool = False, staged: bool = False, ctxs: list | None = None,
                default_stream=None) -> list[Slot]:
    """The `pipeline` slots of a server loop, each with its own context, index, stream and C5 endpoint
    (bench.py's device-resident loop; host_rings / staged for its end-to-end modes)."""
    slots = []
    for i in range(pipeline):
        ctx = ctxs[i] if ctxs and i < len(ctxs) else crk.Context(device_index, **ctx_kw)
        ep = c5_endpoint(ctx, rank, device, n_streams=n_streams, payload_per_stream=payload_per_stream,
                         host_rings=host_rings, staged=staged, h2d_frac=h2d_frac)
        idx = ctx.index(max_rings=n_streams, **INDEX_SHAPE)
        st = torch.cuda.Stream(device) if pipeline > 1 or default_stream is None else default_stream
        slots.append(Slot(ctx, idx, ep, st, crk.PinnedResults(n_streams) if host_rings else None))
    return slots


def run_pipelined(slots: list[Slot], stream, n_steps: int, step_fn=None):
    """bench.py's server loop: step k is served by slot k % P on the slot's stream, so up to P batches are in
    flight.  Returns CUDA events recorded on `stream` before the first and after the last step."""
    P = len(slots)
    step_fn = step_fn or (lambda s: serve_step(s.idx, s.ep, stream=s.stream))
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for s in slots:
        s.stream.wait_event(e0)
    for k in range(n_steps):
        step_fn(slots[k % P])
    for s in slots:
        ev = torch.cuda.Event()
        ev.record(s.stream)
        stream.wait_event(ev)
    e1.record(stream)
    return e0, e1


class StagedLoop:
    """Copy-engine e2e mode (host rings): per slot, inbound DMA (in_stream, after the slot's previous serve
    has read its device rings) -> serve from HBM (stream, after the previous reply DMA has drained the device
    send rings) -> reply DMA (out_stream, queued by the host once the reply sizes are known).  Inbound DMA
    of later batches never waits behind a reply DMA."""

    def __init__(self, slots: list[Slot], device: torch.device, copy_streams: int = 1):
        self.slots = slots
        for s in slots:
            s.in_stream, s.out_stream = torch.cuda.Stream(device), torch.cuda.Stream(device)
            s.in_aux = [torch.cuda.Stream(device) for _ in range(copy_streams - 1)]
            s.out_aux = [torch.cuda.Stream(device) for _ in range(copy_streams - 1)]
            s.ev_in, s.ev_served, s.ev_out = torch.cuda.Event(), torch.cuda.Event(), torch.cuda.Event()
            s.ev_out.record(s.out_stream)
            s.ev_served.record(s.stream)

    @staticmethod
    def _drain(ps: Slot):
        ps.ev_served.synchronize()
        ps.out_stream.wait_event(ps.ev_served)
        staged_out(ps.ep, ps.res.rows(), ps.out_stream, ps.out_aux)
        ps.ev_out.record(ps.out_stream)

    def run(self, n_steps: int):
        P, pend = len(self.slots), []
        for k in range(n_steps):
            s = self.slots[k % P]
            s.in_stream.wait_event(s.ev_served)
            staged_in(s.ep, s.in_stream, s.in_aux)
            s.ev_in.record(s.in_stream)
            s.stream.wait_event(s.ev_in)
            s.stream.wait_event(s.ev_out)
            staged_serve(s.idx, s.ep, s.res, s.stream)
            s.ev_served.record(s.stream)
            pend.append(s)
            if len(pend) >= P:
                self._drain(pend.pop(0))
        for ps in pend:
            self._drain(ps)
        torch.cuda.synchronize()

    def run_mixed(self, n_steps: int):
        """Copy engine in, SM zero-copy out: the inbound window is DMA'd into the device ring, the mover writes
        the replies straight into the pinned host send rings (no outbound DMA)."""
        P = len(self.slots)
        for k in range(n_steps):
            s = self.slots[k % P]
            s.in_stream.wait_event(s.ev_served)
            staged_in(s.ep, s.in_stream)
            s.ev_in.record(s.in_stream)
            s.stream.wait_event(s.ev_in)
            s.idx.serve([(dr, h, t) for dr, (_, h, t) in zip(s.ep.dev_rings, s.ep.rings)], s.ep.sends,
                        s.ep.offs, s.ep.base, s.ep.region.numel(), stream=s.stream)
            s.idx.ring_results_async(s.res, stream=s.stream)
            s.ev_served.record(s.stream)
        torch.cuda.synchronize()

    def run_zero_copy(self, n_steps: int):
        """Zero-copy: the kernels read the CALL rings from and write the reply rings to pinned host memory.
        Step k is launched before the results of step k-1 are read back (device -> host, syncs that slot's
        stream), so the host read overlaps the next batch."""
        P = len(self.slots)
        for k in range(n_steps):
            s = self.slots[k % P]
            serve_step(s.idx, s.ep, stream=s.stream)
            if k >= P - 1:
                p_ = self.slots[(k - P + 1) % P]
                p_.idx.ring_results(len(p_.ep.rings), stream=p_.stream)
        for k in range(max(0, n_steps - P + 1), n_steps):
            p_ = self.slots[k % P]
            p_.idx.ring_results(len(p_.ep.rings), stream=p_.stream)
        torch.cuda.synchronize()


def serve_step(idx: crk.Index, ep: Endpoint, stream=None):
    idx.serve(ep.rings, ep.sends, ep.offs, ep.base, ep.region.numel(), stream=stream)


def staged_in_and_serve(idx: crk.Index, ep: Endpoint, results: "crk.PinnedResults", stream):
    """Copy-engine mode, first half of a step: DMA each host receive window into its device ring,
    serve from HBM into the device send rings, and queue the per-ring results to pinned memory."""
    staged_in(ep, stream)
    staged_serve(idx, ep, results, stream)


def _fan_out(stream, aux):
    """Streams for a step's ring copies: `stream` plus the auxiliary streams, which start after
    everything already queued on `stream`."""
    if not aux:
        return [stream]
    ev = torch.cuda.Event()
    ev.record(stream)
    for a in aux:
        a.wait_event(ev)
    return [stream] + list(aux)


def _fan_in(stream, aux):
    for a in aux or ():
        ev = torch.cuda.Event()
        ev.record(a)
        stream.wait_event(ev)


def staged_in(ep: Endpoint, stream, aux=None):
    """DMA each host receive window into its device ring (ring r on streams[r % n] with aux streams)."""
    ss = _fan_out(stream, aux)
    for r, ((hr, h, t), dr) in enumerate(zip(ep.rings, ep.dev_rings)):
        crk.ring_copy(dr, hr, h, t, stream=ss[r % len(ss)])
    _fan_in(stream, aux)


def staged_serve(idx: crk.Index, ep: Endpoint, results: "crk.PinnedResults", stream):
    """Serve the staged device rings into the device send rings; queue the per-ring results."""
    idx.serve([(dr, h, t) for dr, (_, h, t) in zip(ep.dev_rings, ep.rings)], ep.dev_sends, ep.offs, ep.base,
              ep.region.numel(), stream=stream)
    idx.ring_results_async(results, stream=stream)


def staged_out(ep: Endpoint, rows: list, stream, aux=None):
    """Second half: DMA each ring's reply bytes (now known on the host) back to the host send ring."""
    ss = _fan_out(stream, aux)
    for r, (hs, ds, off) in enumerate(zip(ep.sends, ep.dev_sends, ep.offs)):
        n = rows[r]["reply_bytes"]
        if n:
            crk.ring_copy(hs, ds, off, off + n, stream=ss[r % len(ss)])
    _fan_in(stream, aux)


def check_results(idx: crk.Index, ep: Endpoint) -> dict:
    """Cheap end-of-run sanity on the device results: every ring consumed, every record OK, reply bytes
    as the closed forms predict, and a sample of HtoD destinations equal to the generator's payload."""
    res = idx.ring_results(len(ep.rings))
    ok = all(r["status"] == crk.OK and r["consumed"] == t for r, (_, _, t) in zip(res, ep.rings))
    ok &= all(r["n_records"] == n for r, n in zip(res, ep.per_stream_records))
    ok &= all(r["reply_bytes"] == w for r, w in zip(res, ep.per_stream_reply))
    sampled = 0
    for s in ep.streams[:2]:
        for r in [x for x in s.records if x.kind == gen.PROC_H2D][:3]:
            want = torch.from_numpy(gen.random_bytes(r.seed & 0xFFFFFFFF, r.size)).to(ep.region.device)
            ok &= bool(torch.equal(ep.region[r.region_off:r.region_off + r.size], want))
            sampled += 1
    return dict(ok=bool(ok), sampled_h2d_records=sampled)


# ------------------------------------------------------------------ host-link sweeps (C3, C2) through host rings

class LinkSweep:
    """bandwidthTest-shaped end-to-end runs through pinned host rings:
    one memcpy CALL of n bytes per run, HtoD (the CALL carries the payload; the 32-byte REPLY goes back) or DtoH
    (a 64-byte CALL; the framed payload REPLY goes back), `slots` calls in flight (consecutive calls alternate
    between slots, so one call's copies overlap the previous call's kernels).  Two ways to serve a call:
      ce: crk_ring_copy DMAs the receive window into a device ring, crk_serve runs from HBM into a device send
          ring, crk_ring_copy DMAs the reply bytes out (copy engines for the host link);
      zc: crk_serve reads the pinned receive ring and writes the pinned send ring over the link (zero-copy).
    Every run includes the host -> device copy of its CALL and the device -> host copy of its REPLY; the times
    are CUDA events on the launching streams around all runs of a size."""

    def __init__(self, device_index: int, device: torch.device, max_n: int = 1 << 30, slots: int = 2, **ctx_kw):
        # one context per slot: a context's scratch serves one call at a time (include/crk.h)
        ctxs = [crk.Context(device_index, **ctx_kw) for _ in range(slots)]
        self.ctx, self.dev, F = ctxs[0], device, ctxs[0].cfg.frag_payload
        self.big = next_pow2(max_n + 64 + 4 * (max_n // F + 2))  # a ring for the larger side of any call
        self.slots = []
        for ctx in ctxs:
            sl = type("SweepSlot", (), {})()
            sl.ctx = ctx
            sl.host_big = crk.Ring.host(self.big)
            sl.host_small = crk.Ring.host(4096)
            sl.dev_big = crk.Ring.device(self.big, device)
            sl.dev_small = crk.Ring.device(4096, device)
            sl.region = torch.zeros(max_n + 256, dtype=torch.uint8, device=device)
            sl.idx = None  # sized per call by prepare / prepare_c2
            sl.stream, sl.in_s, sl.out_s = (torch.cuda.Stream(device) for _ in range(3))
            sl.ev_in, sl.ev_served, sl.ev_out = torch.cuda.Event(), torch.cuda.Event(), torch.cuda.Event()
            self.slots.append(sl)

    def _sub(self, ring: crk.Ring, cap: int) -> crk.Ring:
        return ring.sub(0, cap)

    def prepare(self, n: int, direction: str, payload: torch.Tensor):
        """Encodes the CALL of each slot (setup, outside the timed region): HtoD carries `payload`, DtoH reads it
        from the slot's region."""
        F = self.ctx.cfg.frag_payload
        self.n, self.direction = n, direction
        for i, sl in enumerate(self.slots):
            base = sl.region.data_ptr()
            # an index sized for the call, as a server sizes its buffers for its calls: a small one (up to
            # crk_config.fused_front_max_frags fragments) lets crk_serve take the fused single-CTA front end
            sl.idx = sl.ctx.index(1, n // F + 64, 16)
            if direction == "h2d":
                stage = self._sub(sl.dev_big, self.big)
                w = sl.ctx.encode_call(0x5E0000 + i, gen.PROC_H2D, [(crk.K_U64, base), (crk.K_OPAQUE_VAR, payload),
                                                                     (crk.K_U64, n)], stage, 0)
                torch.cuda.synchronize(self.dev)
                crk.ring_copy(sl.host_big, sl.dev_big, 0, w)
                sl.rx_host, sl.rx_dev, sl.w_in = sl.host_big, sl.dev_big, w
                sl.tx_host, sl.tx_dev, sl.w_out = sl.host_small, sl.dev_small, crk.wire_size_d2h(0, 1, F)
            else:
                sl.region[:n].copy_(payload)
                w = sl.ctx.encode_call(0x5D0000 + i, gen.PROC_D2H, [(crk.K_U64, base), (crk.K_U64, n)], sl.dev_small, 0)
                torch.cuda.synchronize(self.dev)
                crk.ring_copy(sl.host_small, sl.dev_small, 0, w)
                sl.rx_host, sl.rx_dev, sl.w_in = sl.host_small, sl.dev_small, w
                sl.tx_host, sl.tx_dev, sl.w_out = sl.host_big, sl.dev_big, crk.wire_size_d2h(n, 0, F)
            sl.ev_served.record(sl.stream)
            sl.ev_out.record(sl.out_s)
        torch.cuda.synchronize(self.dev)

    def prepare_c2(self):
        """The matrixMul batch: A (409,600 B of 1.0f) and B (819,200 B of 0.01f)
        HtoD and C (819,200 B of 3.2f) DtoH, three CALLs served as one batch; wire in 1,229,060 B, out 819,348 B."""
        F = self.ctx.cfg.frag_payload
        A, B, Cm = (torch.from_numpy(x.view(np.uint8).copy()).to(self.dev) for x in gen.c2_matrices())
        self.direction, self.c2 = "c2", (A, B, Cm)
        half = self.big // 2
        for i, sl in enumerate(self.slots):
            base = sl.region.data_ptr()
            sl.idx = sl.ctx.index(1, (1 << 21) // F + 64, 16)
            offA, offB, offC = 0, 409_600, 409_600 + 819_200
            sl.region[offC:offC + Cm.numel()].copy_(Cm)
            rx_dev, tx_dev = sl.dev_big.sub(0, 1 << 21), sl.dev_big.sub(half, 1 << 20)
            rx_host, tx_host = sl.host_big.sub(0, 1 << 21), sl.host_big.sub(half, 1 << 20)
            w = 0
            for xid, kind, items in ((0xC2A, gen.PROC_H2D, [(crk.K_U64, base + offA), (crk.K_OPAQUE_VAR, A),
                                                            (crk.K_U64, A.numel())]),
                                     (0xC2B, gen.PROC_H2D, [(crk.K_U64, base + offB), (crk.K_OPAQUE_VAR, B),
                                                            (crk.K_U64, B.numel())]),
                                     (0xC2C, gen.PROC_D2H, [(crk.K_U64, base + offC), (crk.K_U64, Cm.numel())])):
                w += sl.ctx.encode_call(xid, kind, items, rx_dev, w)
            torch.cuda.synchronize(self.dev)
            crk.ring_copy(rx_host, rx_dev, 0, w)
            sl.rx_host, sl.rx_dev, sl.w_in = rx_host, rx_dev, w
            sl.tx_host, sl.tx_dev = tx_host, tx_dev
            sl.w_out = 2 * crk.wire_size_d2h(0, 1, F) + crk.wire_size_d2h(Cm.numel(), 0, F)
            sl.ev_served.record(sl.stream)
            sl.ev_out.record(sl.out_s)
        torch.cuda.synchronize(self.dev)

    def run(self, mode: str, runs: int, main) -> float:
        """`runs` calls in `mode` ("ce" / "zc"); returns device ms over all of them (events on `main`)."""
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(main)
        for sl in self.slots:
            for st in (sl.stream, sl.in_s, sl.out_s):
                st.wait_event(e0)
        for k in range(runs):
            sl = self.slots[k % len(self.slots)]
            base, nb = sl.region.data_ptr(), sl.region.numel()
            if mode == "ce":
                sl.in_s.wait_event(sl.ev_served)
                crk.ring_copy(sl.rx_dev, sl.rx_host, 0, sl.w_in, stream=sl.in_s)
                sl.ev_in.record(sl.in_s)
                sl.stream.wait_event(sl.ev_in)
                sl.stream.wait_event(sl.ev_out)
                sl.idx.serve([(sl.rx_dev, 0, sl.w_in)], [sl.tx_dev], [0], base, nb, stream=sl.stream)
                sl.ev_served.record(sl.stream)
                sl.out_s.wait_event(sl.ev_served)
                crk.ring_copy(sl.tx_host, sl.tx_dev, 0, sl.w_out, stream=sl.out_s)
                sl.ev_out.record(sl.out_s)
            else:
                sl.idx.serve([(sl.rx_host, 0, sl.w_in)], [sl.tx_host], [0], base, nb, stream=sl.stream)
        for sl in self.slots:
            for st in (sl.stream, sl.in_s, sl.out_s):
                ev = torch.cuda.Event()
                ev.record(st)
                main.wait_event(ev)
        e1.record(main)
        torch.cuda.synchronize(self.dev)
        return e0.elapsed_time(e1)

    def check(self, payload: torch.Tensor) -> bool:
        """Every slot's last call served OK: HtoD destinations == payload; DtoH: the reply's size and, past its
        first fragment header and the 32-byte REPLY prefix, the payload's first bytes."""
        ok = True
        for sl in self.slots:
            r = sl.idx.ring_results(1)[0]
            ok &= r["status"] == crk.OK and r["reply_bytes"] == sl.w_out
            if self.direction == "c2":
                A, B, Cm = self.c2
                ok &= bool(torch.equal(sl.region[:A.numel()], A)) and bool(
                    torch.equal(sl.region[409_600:409_600 + B.numel()], B))
                # C's reply follows the two 32-byte HtoD replies: its payload starts 36 bytes in
                ok &= sl.tx_host.read(64 + 36, 1024) == bytes(Cm[:1024].cpu().numpy())
            elif self.direction == "h2d":
                ok &= bool(torch.equal(sl.region[:self.n], payload))
            else:
                k = min(self.n, 1024)
                ok &= sl.tx_host.read(36, k) == bytes(payload[:k].cpu().numpy())
        return bool(ok)
