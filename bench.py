#!/usr/bin/env python
"""Benchmark: XDR memcpy decode/encode GB/s per GPU (and aggregate over N GPUs) vs the binding roofline.

Workload (BASELINE.json configs[4], the per-GPU slice of the metric's 8-GPU aggregate): one Cricket
server endpoint per GPU serving 16 client streams, each a ring of ONC RPC memcpy CALL records (sizes
log-uniform 4 KiB-16 MiB, 50/50 HtoD/DtoH, 64 MiB of payload per stream = 1 GiB per GPU), fragments of
64 KiB.  One step = crk_serve over all 16 rings: record-marking scan (K1), prefix
sums (K2), CALL parse (K3), HtoD opaque scatter into device memory (K4) and DtoH reply encode into the
send rings (K6), i.e. every §8(a) row the memcpy path has.

  value : payload GB/s (1e9 B/s) with rings and send rings resident in HBM (inputs > L2: 1 GiB of rings),
          3 batches in flight
  e2e   : the same through the C ABI with the receive and send rings in pinned host memory, plus a
          device->host read of the per-ring results every step; the fastest of three modes (copy-engine
          staged, mixed, zero-copy), each measured, against the host link measured in the same run
  roofline: the mover kernel (K4/K6) against the measured HBM copy bandwidth (per launch, and over the
          timed region)
  cpu_baseline: the oracle (oracle/, plain C) on a bounded sample of the same workload: one core, one
          thread per core, and Cricket-style (pageable buffer + cudaMemcpy)
  --direction h2d|d2h: the HtoD-only / DtoH-only call mixes of the same endpoint

Launch: python bench.py [--gpus N --steps K --warmup W]; N > 1 under torch.distributed.run (one rank per
GPU; a CPU gloo group for the barrier and the max-over-ranks of the timings -- no NCCL: the data path has no
collective).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

MiB = 1 << 20


def parse_args():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=200)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="crk", choices=["crk", "reference"])
    p.add_argument("--streams", type=int, default=16)
    p.add_argument("--payload-mib", type=int, default=64, help="payload per stream")
    p.add_argument("--e2e-steps", type=int, default=100)
    p.add_argument("--pipeline", type=int, default=3, help="batches in flight (server loop slots)")
    p.add_argument("--e2e-pipeline", type=int, default=3, help="batches in flight for the host-memory runs")
    p.add_argument("--e2e-copy-streams", type=int, default=1, help="streams per direction for the staged ring DMAs")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-sweep", action="store_true", help="skip the C3 / C2 host-link sweeps")
    p.add_argument("--sweep-log2", default="12-30", help="C3 sweep sizes as log2 range, e.g. 12-30")
    p.add_argument("--no-cpu", action="store_true")
    p.add_argument("--cpu-seconds", type=float, default=10.0)
    p.add_argument("--ctx", default="", help="crk_config overrides, e.g. scan_threads=128,tile_bytes=32768")
    p.add_argument("--e2e-ctx", default="", help="extra crk_config overrides for the host-ring (e2e) contexts")
    p.add_argument("--direction", default="mixed", choices=["mixed", "h2d", "d2h"],
                   help="C5 call mix: 50/50 (default), HtoD-only or DtoH-only memcpys")
    return p.parse_args()


# ------------------------------------------------------------------ clocks during the timed region

class ClockSampler:
    """NVML sampling of SM clocks and throttle reasons on a background thread."""

    def __init__(self, index: int, period_s: float = 0.002):
        self.index, self.period, self.samples, self.reasons = index, period_s, [], set()
        self._stop = threading.Event()
        self.max_mhz = None
        try:
            import pynvml as N
            N.nvmlInit()
            self.N = N
            self.h = N.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = N.nvmlDeviceGetMaxClockInfo(self.h, N.NVML_CLOCK_SM)
        except Exception as e:  # pragma: no cover
            self.N = None
            self.err = repr(e)

    def _run(self):
        N = self.N
        names = {getattr(N, k, None): k for k in (
            "nvmlClocksEventReasonHwSlowdown", "nvmlClocksEventReasonHwThermalSlowdown",
            "nvmlClocksEventReasonSwThermalSlowdown", "nvmlClocksEventReasonSwPowerCap",
            "nvmlClocksEventReasonHwPowerBrakeSlowdown")}
        label = {"nvmlClocksEventReasonHwSlowdown": "hw_slowdown",
                 "nvmlClocksEventReasonHwThermalSlowdown": "hw_thermal_slowdown",
                 "nvmlClocksEventReasonSwThermalSlowdown": "sw_thermal_slowdown",
                 "nvmlClocksEventReasonSwPowerCap": "sw_power_cap",
                 "nvmlClocksEventReasonHwPowerBrakeSlowdown": "hw_power_brake"}
        while not self._stop.is_set():
            try:
                self.samples.append(N.nvmlDeviceGetClockInfo(self.h, N.NVML_CLOCK_SM))
                r = N.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, k in names.items():
                    if bit and r & bit:
                        self.reasons.add(label[k])
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.N:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.N:
            self._stop.set()
            self.t.join()

    def summary(self):
        if not self.N:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "error": getattr(self, "err", "")}
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None, "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ------------------------------------------------------------------ CPU baseline (oracle)

def oracle_sample(stream_ids, payload_mib: int, rank: int = 0):
    """Oracle-encoded rings for streams `stream_ids` of endpoint `rank` (a bounded sample of the workload),
    with a host region of their own (their destinations / sources rebased to its start)."""
    import numpy as np
    import oracle as O
    from paper_conf_sc_eilingkkflm23_b200 import gen
    streams, _ = gen.c5_endpoint(rank, n_streams=16, payload_per_stream=payload_mib * MiB,
                                 h2d_budget=payload_mib * MiB - payload_mib * MiB // 16)
    cfg = O.Config(prog=gen.PROG, vers=gen.VERS, proc_h2d=gen.PROC_H2D, proc_d2h=gen.PROC_D2H, frag_payload=65536)
    base = 0x7F0000000000
    sample = [streams[i] for i in stream_ids]
    lo = min(r.region_off for s in sample for r in s.records) & ~255
    top = max(r.region_off + r.size for s in sample for r in s.records) - lo
    region = np.zeros(top + 256, np.uint8)
    rings, send_caps, payload = [], [], 0
    for s in sample:
        wires, reply = [], 0
        for r in s.records:
            d = gen.random_bytes(r.seed & 0xFFFFFFFF, r.size)
            payload += r.size
            off = r.region_off - lo
            if r.kind == gen.PROC_H2D:
                wires.append(O.encode_call(r.xid, r.kind, [(O.K_U64, base + off), (O.K_OPAQUE_VAR, d),
                                                           (O.K_U64, r.size)], cfg))
                reply += 64
            else:
                region[off:off + r.size] = d
                wires.append(O.encode_call(r.xid, r.kind, [(O.K_U64, base + off), (O.K_U64, r.size)], cfg))
                reply += r.size + 64 + 4 * (r.size // 65536 + 1)
        w = b"".join(wires)
        cap = 1 << max(8, len(w).bit_length())
        ring = np.zeros(cap, np.uint8)
        ring[:len(w)] = np.frombuffer(w, np.uint8)
        rings.append((ring, 0, len(w)))
        send_caps.append(1 << max(8, reply.bit_length()))

    def step():
        out = O.serve(rings, cfg, region, base, send_caps, [0] * len(rings), max_frags_per_ring=1 << 16,
                      max_records_per_ring=1 << 12)
        assert all(s == O.OK for s in out["scan_status"])
        return out

    return step, payload, region


def _timed_loop(step, seconds: float):
    step()  # warm (page-in)
    t0 = time.perf_counter()
    reps = 0
    while True:
        step()
        reps += 1
        el = time.perf_counter() - t0
        if el >= seconds:
            return reps, el


def cpu_baseline(args, seconds: float):
    """The oracle as it stands, on this box's host cores (SURVEY.md §8(d) "Oracle (CPU baseline)"):
    (i) one thread -- the analogue of Cricket's single-core RPC path -- is `value`;
    (ii) one thread per core over independent client streams (ctypes releases the GIL in or_serve);
    (iii) Cricket-style: decode into a pageable host buffer, then cudaMemcpy it to the device."""
    import torch
    n_streams = 2
    step, payload, _ = oracle_sample(list(range(n_streams)), args.payload_mib)
    reps, el = _timed_loop(step, seconds)
    out = {"value": round(payload * reps / el / 1e9, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
           "sample": f"oracle or_serve (plain C, 1 thread) over streams 0-{n_streams - 1} of endpoint 0 "
                     f"({payload / MiB:.0f} MiB payload) x{reps} reps, {el:.1f} s"}
    try:
        import platform
        out["cpu_model"] = next((l.split(":", 1)[1].strip() for l in open("/proc/cpuinfo")
                                 if l.startswith("model name")), platform.processor())
    except OSError:
        pass
    # (ii) one thread per core, each serving its own stream (own ring, region and send ring)
    nthr = max(1, min(len(os.sched_getaffinity(0)), 16))  # the cores bench.py is bound to (GPU NUMA node)
    samples = [oracle_sample([t], args.payload_mib) for t in range(nthr)]
    for st, _, _ in samples:
        st()
    done = [0] * nthr
    stop_at = time.perf_counter() + seconds / 2

    def worker(i):
        while time.perf_counter() < stop_at:
            samples[i][0]()
            done[i] += 1

    t0 = time.perf_counter()
    ths = [threading.Thread(target=worker, args=(i,)) for i in range(nthr)]
    for t in ths:
        t.start()
    for t in ths:
        t.join()
    el = time.perf_counter() - t0
    moved = sum(done[i] * samples[i][1] for i in range(nthr))
    out["threads"] = {"value": round(moved / el / 1e9, 4), "unit": "GB/s", "cores": nthr,
                      "sample": f"{nthr} threads, thread t serves stream t of endpoint 0 alone "
                                f"({args.payload_mib} MiB payload each), {sum(done)} stream-steps in {el:.1f} s"}
    del samples
    # (iii) Cricket-style: DtoH sources cudaMemcpy'd into the pageable host region, the oracle decodes and
    # encodes there, then the region (HtoD destinations) is cudaMemcpy'd back to the device
    if torch.cuda.is_available():
        dev = torch.device("cuda", torch.cuda.current_device())
        step3, payload3, region = oracle_sample(list(range(n_streams)), args.payload_mib)
        host = torch.from_numpy(region)
        d_region = host.to(dev)

        def cricket_step():
            host.copy_(d_region)   # pageable D2H
            step3()
            d_region.copy_(host)   # pageable H2D
            torch.cuda.synchronize(dev)

        reps, el = _timed_loop(cricket_step, seconds / 2)
        out["cricket_style"] = {"value": round(payload3 * reps / el / 1e9, 4), "unit": "GB/s", "cores": 1,
                                "sample": f"oracle or_serve into a pageable host buffer + cudaMemcpy of the "
                                          f"{region.size / MiB:.0f} MiB region each way, streams 0-{n_streams - 1}, "
                                          f"x{reps} reps, {el:.1f} s"}
        del d_region
    return out


def run_reference(args):
    """--impl reference: the oracle timed as the reference arm (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    n_streams = 2
    step, payload, _ = oracle_sample(list(range(n_streams)), args.payload_mib)
    for _ in range(args.warmup):
        step()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        step()
    el = time.perf_counter() - t0
    v = payload * args.steps / el / 1e9
    sample = (f"oracle or_serve (plain C, 1 thread) over streams 0-{n_streams - 1} of endpoint 0 "
              f"({payload / MiB:.0f} MiB payload per step)")
    print(json.dumps({
        "impl": "reference", "metric": "xdr_memcpy_serve_payload_GBps", "value": round(v, 4), "unit": "GB/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(el / args.steps * 1e3, 3),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": workload_config(args), "cpu_baseline": {"value": round(v, 4), "unit": "GB/s", "cores": 1,
                                                           "kind": "oracle", "sample": sample},
        "e2e": {"value": round(v, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}))


H2D_FRAC = {"mixed": 0.5, "h2d": 1.0, "d2h": 0.0}


def workload_config(args):
    mix = {"mixed": "50/50 HtoD/DtoH", "h2d": "HtoD only", "d2h": "DtoH only"}[args.direction]
    return {"workload": f"C5 endpoint per GPU: {args.streams} client streams x {args.payload_mib} MiB memcpy payload "
                        f"(ONC RPC CALLs, sizes log-uniform 4 KiB-16 MiB, {mix}, F=64 KiB fragments)",
            "direction": args.direction,
            "streams_per_gpu": args.streams, "payload_per_gpu_bytes": args.streams * args.payload_mib * MiB,
            "frag_payload": 65536, "l2": "inputs larger than L2 (rings + region > 2 GiB per GPU)",
            "parallelism": f"{args.gpus} independent endpoints, no collective"}


# ------------------------------------------------------------------ main

def main():
    args = parse_args()
    if args.impl == "reference":
        run_reference(args)
        return
    import torch
    import torch.distributed as dist
    from paper_conf_sc_eilingkkflm23_b200 import build, crk, parallel, workload

    world, rank, local = parallel.rank_env()
    ndev = torch.cuda.device_count()
    local = local % ndev  # more ranks than GPUs (plumbing runs): ranks share devices
    parallel.init(world)  # gloo on the CPU: barrier + timing reductions only, no NCCL (north_star)
    torch.cuda.set_device(local)
    dev = torch.device(f"cuda:{local}")
    numa = parallel.bind_numa(local)  # before any pinned host allocation
    red_dev = "cpu"
    build.build()

    ctx_kw = {k: int(v, 0) for k, v in (kv.split("=") for kv in args.ctx.split(",") if kv)}

    def barrier():
        parallel.barrier(dev)

    def max_over_ranks(x: float) -> float:
        return parallel.max_over_ranks(x, red_dev)

    def sum_over_ranks(x: float) -> float:
        return parallel.sum_over_ranks(x, red_dev)

    # A server loop keeps `pipeline` batches in flight: each slot is a (context, index, stream, batch
    # buffers) set, so the front end (scan / parse / plan) of batch k+1 runs while the mover of batch k
    # streams bytes.  Step k is served by slot k % pipeline; every step is one full pass over its batch.
    # workload.run_pipelined / StagedLoop are the loops timed here; tests/test_gpu_bench_parity.py runs the
    # same functions on the same configuration and compares every byte with the oracle.
    P = max(1, args.pipeline)
    ctx_kw = workload.pipelined_ctx_kw(ctx_kw, P)
    stream = torch.cuda.current_stream(dev)
    slots = workload.build_slots(local, rank, dev, P, ctx_kw, n_streams=args.streams,
                                 payload_per_stream=args.payload_mib * MiB, h2d_frac=H2D_FRAC[args.direction],
                                 default_stream=stream)
    ep = slots[0].ep

    def run(n_steps):
        return workload.run_pipelined(slots, stream, n_steps)

    # ---- device-resident timed region (value)
    run(max(args.warmup, P))
    barrier()
    check = workload.check_results(slots[0].idx, slots[0].ep)
    l0 = crk.kernel_launches()
    barrier()
    with ClockSampler(local) as clk:
        torch.cuda.profiler.start()  # the timed region is the profiler window (ncu --profile-from-start off)
        e0, e1 = run(args.steps)
        torch.cuda.synchronize()
        torch.cuda.profiler.stop()
    launches = crk.kernel_launches() - l0
    ms = e0.elapsed_time(e1) / args.steps
    ms_max = max_over_ranks(ms)
    payload_all = sum_over_ranks(ep.payload)
    value = payload_all / (ms_max / 1e3) / 1e9
    # The same steps one batch at a time (no overlap between batches): the per-stage CUDA-event times,
    # and the dominant kernel's launch time for the roofline, are taken here, where a launch's events
    # bracket only its own execution (in the pipelined pass a launch also waits for the previous batch's
    # mover to leave the SMs).
    s0 = slots[0]
    n_serial = min(args.steps, 50)
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)

    def serial_ms_of(idx):  # one batch at a time, no stage events (they would sit between the kernels)
        f0.record(s0.stream)
        for _ in range(n_serial):
            workload.serve_step(idx, s0.ep, stream=s0.stream)
        f1.record(s0.stream)
        torch.cuda.synchronize()
        return max_over_ranks(f0.elapsed_time(f1) / n_serial)

    serial_ms = serial_ms_of(s0.idx)
    crk.profile_enable(True)  # the same steps again with the stage events
    for _ in range(n_serial):
        workload.serve_step(s0.idx, s0.ep, stream=s0.stream)
    torch.cuda.synchronize()
    prof = crk.profile_read()
    crk.profile_enable(False)
    # The same batch served alone by a context with the library defaults (the chunked multi-CTA scan for
    # long windows, the whole grid for the mover): a single batch's latency and its stage shares.
    ctx_l = crk.Context(local)
    idx_l = ctx_l.index(max_rings=args.streams, **workload.INDEX_SHAPE)
    for _ in range(3):
        workload.serve_step(idx_l, s0.ep, stream=s0.stream)
    torch.cuda.synchronize()
    lone_ms = serial_ms_of(idx_l)  # latency without the stage events (which would break the PDL chaining)
    crk.profile_enable(True)
    for _ in range(n_serial):
        workload.serve_step(idx_l, s0.ep, stream=s0.stream)
    torch.cuda.synchronize()
    prof_l = crk.profile_read()
    crk.profile_enable(False)
    lone = {"ms_per_step": round(lone_ms, 4),
            "stages_ms_per_step": {k: round(v[0] / max(1, v[1]), 4) for k, v in prof_l.items()},
            "stage_share": {k: round(v[0] / max(1e-9, sum(x[0] for x in prof_l.values())), 4)
                            for k, v in prof_l.items()},
            "scan_stats": idx_l.scan_stats(),
            "config": "library defaults (chunked multi-CTA scan of long windows, whole-grid mover), one batch "
                      "at a time"}
    lone["value"] = round(sum_over_ranks(ep.payload) / (lone["ms_per_step"] / 1e3) / 1e9, 2)
    del idx_l, ctx_l

    # roofline of the dominant kernel (the mover): algorithmic HBM bytes per launch / its event time
    mv_ms, mv_n = prof["move"]
    alg_bytes = 2 * ep.h2d_payload + ep.d2h_payload + ep.reply_wire  # read+write per HtoD byte; DtoH read + reply
    mv_launch_ms = mv_ms / max(1, mv_n)
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    hbm_peak = float(peaks.get("hbm_gbs", 6650.0))
    achieved = alg_bytes / (mv_launch_ms / 1e3) / 1e9
    traffic = None
    try:
        traffic = json.load(open(os.path.join(ROOT, "profiles", "mover_ncu.json")))["dram_bytes_per_launch"]
    except Exception:
        pass
    stage_share = {k: round(v[0] / max(1e-9, sum(x[0] for x in prof.values())), 4) for k, v in prof.items()}

    # ---- end to end through the C ABI with host (pinned, mapped) rings
    e2e = None
    if not args.no_e2e:
        ctxs = [s.ctx for s in slots]
        del slots
        e2e_kw = {k: int(v, 0) for k, v in (kv.split("=") for kv in args.e2e_ctx.split(",") if kv)}
        if e2e_kw:  # contexts of their own for the host-ring runs
            ctxs = [crk.Context(local, **{**ctx_kw, **e2e_kw}) for _ in range(max(1, args.e2e_pipeline))]
        torch.cuda.empty_cache()
        # host-link peaks (copy engine, pinned) measured before the rings are allocated (their buffers get
        # the same placement the rings get) and again after the runs; the roofline takes the better of the two.
        # Every rank measures at the same time (after a barrier): with N GPUs the links share the host.
        barrier()
        link0 = host_link_peaks(dev)
        P = max(1, args.e2e_pipeline)  # batches in flight for the host-memory runs
        hslots = workload.build_slots(local, rank, dev, P, {**ctx_kw, **e2e_kw}, n_streams=args.streams,
                                      payload_per_stream=args.payload_mib * MiB, h2d_frac=H2D_FRAC[args.direction],
                                      host_rings=True, staged=True, ctxs=ctxs, default_stream=stream)
        ep_h = hslots[0].ep
        loop = workload.StagedLoop(hslots, dev, args.e2e_copy_streams)
        run_staged, run_mixed, run_e2e = loop.run, loop.run_mixed, loop.run_zero_copy

        run_staged(max(2, min(args.warmup, 4)))
        barrier()
        t0 = time.perf_counter()
        run_staged(args.e2e_steps)
        el_st = max_over_ranks(time.perf_counter() - t0)
        rows = hslots[0].res.rows()
        check_st = workload.check_results(hslots[0].idx, ep_h)
        n0 = rows[0]["reply_bytes"]
        check_st["host_send_matches_device"] = bool(
            hslots[0].ep.sends[0].read(0, n0) == hslots[0].ep.dev_sends[0].read(0, n0))
        check_st["ok"] = check_st["ok"] and check_st["host_send_matches_device"]

        run_mixed(max(2, min(args.warmup, 4)))
        barrier()
        t0 = time.perf_counter()
        run_mixed(args.e2e_steps)
        el_mx = max_over_ranks(time.perf_counter() - t0)
        check_mx = workload.check_results(hslots[0].idx, ep_h)

        run_e2e(max(2, min(args.warmup, 4)))
        barrier()
        t0 = time.perf_counter()
        run_e2e(args.e2e_steps)
        el = time.perf_counter() - t0
        el_max = max_over_ranks(el)
        check_h = workload.check_results(hslots[0].idx, ep_h)
        res_bytes = len(ep_h.rings) * 40
        e2e_v = sum_over_ranks(ep_h.payload) * args.e2e_steps / el_max / 1e9
        # live host-link peaks (copy engine, pinned) for the e2e roofline
        barrier()
        link1 = host_link_peaks(dev)
        link = {k: max(link0[k], link1[k]) for k in link0}
        link["measured"] = ("best of two measurements (before allocating the rings, after the runs), every rank "
                            "at once after a barrier")
        link["before"], link["after"] = link0, link1
        links = parallel.gather({k: link[k] for k in link0})
        wires = parallel.gather((ep_h.wire_in, ep_h.reply_wire))
        link_job = parallel.link_aggregate(links)
        t_link = max(ep_h.wire_in / link["ce_h2d_gbs"], ep_h.reply_wire / link["ce_d2h_gbs"],
                     (ep_h.wire_in + ep_h.reply_wire) / link["ce_bidir_gbs"]) / 1e9
        del hslots, loop
        torch.cuda.empty_cache()
        barrier()
        shaped_ms = shaped_link_ms(dev, ep_h.wire_in, ep_h.reply_wire)
        modes = []
        for name, el_m, chk in (
                (f"zero-copy: kernels read CALL rings from and write reply rings to pinned host memory; "
                 f"{P} batches in flight", el_max, check_h),
                (f"copy-engine staged: crk_ring_copy DMAs each receive window into a device ring, crk_serve "
                 f"decodes from HBM into device send rings, crk_ring_copy DMAs the replies back; {P} batches in "
                 f"flight", el_st, check_st),
                (f"mixed: crk_ring_copy DMAs each receive window into a device ring, crk_serve decodes from HBM "
                 f"and the mover writes the replies straight into the pinned host send rings; {P} batches in "
                 f"flight", el_mx, check_mx)):
            step_s = el_m / args.e2e_steps
            modes.append({"value": round(sum_over_ranks(ep_h.payload) / step_s / 1e9, 3), "unit": "GB/s",
                          "h2d_bytes_per_step": ep_h.wire_in, "d2h_bytes_per_step": ep_h.reply_wire + res_bytes,
                          "ms_per_step": round(step_s * 1e3, 3), "mode": name,
                          "wire_gbs": round((ep_h.wire_in + ep_h.reply_wire) / step_s / 1e9, 3),
                          "host_link": {**link, "pcie_gen5_x16_theoretical_gbs": 63.0,
                                        # the tighter of the two measured bounds: the LP bound of the copy-engine
                                        # rates, and the copy engines moving exactly this step's bytes both ways
                                        # at once (a box whose short bidirectional probe under-reads the link
                                        # would otherwise give a fraction above 1)
                                        "bound_ms": round(min(t_link * 1e3, shaped_ms), 3),
                                        "frac": round(min(t_link, shaped_ms / 1e3) / step_s, 4),
                                        "bound_lp_ms": round(t_link * 1e3, 3),
                                        "frac_lp": round(t_link / step_s, 4),
                                        "shaped_bound_ms": round(shaped_ms, 3),
                                        "frac_shaped": round(shaped_ms / 1e3 / step_s, 4),
                                        "shaped_how": "the copy engines alone moving this step's wire bytes in "
                                                      "and out at the same time (shaped_link_ms)",
                                        "job": {**link_job, **parallel.link_bound_frac(links, wires, step_s)}},
                          "check": chk})
        modes.sort(key=lambda m: -m["value"] if m["check"]["ok"] else 0)
        e2e = dict(modes[0])
        e2e["other_modes"] = [{k: m[k] for k in ("value", "mode", "ms_per_step", "check")} for m in modes[1:]]
        del ep_h
        torch.cuda.empty_cache()
    sweep = None
    if not args.no_sweep and rank == 0:  # one GPU's curve (the others idle at the final barrier)
        if e2e is None:
            link = host_link_peaks(dev)
        sweep = run_sweep(args, dev, link)

    out = {
        "metric": "xdr_memcpy_serve_payload_GBps", "value": round(value, 2), "unit": "GB/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_max, 4), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u8",
        "data": "synthetic (seeded gen.c5_endpoint; CALLs encoded on the GPU by crk_rpc_encode_call)",
        "config": workload_config(args),
        "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": hbm_peak, "unit": "GB/s",
                     "frac": round(achieved / hbm_peak, 4), "traffic": traffic,
                     "kernel": "crk mover_kernel (K4 opaque scatter + K6 reply encode)",
                     "alg_bytes_per_launch": alg_bytes, "launch_ms": round(mv_launch_ms, 4),
                     "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy, read+write)",
                     "measured": "CUDA events around each mover launch in the serial pass of this run "
                                 "(same contexts and launch configuration as the timed region)",
                     "in_timed_region": {"achieved": round(alg_bytes / (ms_max / 1e3) / 1e9, 1),
                                         "frac": round(alg_bytes / (ms_max / 1e3) / 1e9 / hbm_peak, 4),
                                         "how": "mover algorithmic bytes per step / ms_per_step of the pipelined "
                                                "timed region (a lower bound: the step also holds scan/parse/plan)"},
                     "mover_config": {k: ctx_kw.get(k) for k in ("mover_reserve_ctas", "mover_tail_tiles", "mover_run")}},
        "wire_gbs": round(sum_over_ranks(ep.wire_in + ep.reply_wire) / (ms_max / 1e3) / 1e9, 2),
        "pipeline": P, "serial_ms_per_step": round(serial_ms, 4), "lone_batch": lone,
        "serial_value": round(payload_all / (serial_ms / 1e3) / 1e9, 2),
        "stages_ms_per_step": {k: round(v[0] / max(1, v[1]), 4) for k, v in prof.items()},
        "stage_share": stage_share,
        "payload_bytes_per_gpu": ep.payload, "wire_in_bytes_per_gpu": ep.wire_in,
        "reply_bytes_per_gpu": ep.reply_wire, "records_per_gpu": ep.n_records,
        "gpu_launches": launches, "check": check, "host_numa": numa,
        "clocks": clk.summary(),
        "e2e": e2e,
        "sweep": sweep,
    }
    if rank == 0 and not args.no_cpu:  # rank 0 only, after every rank's timed regions
        out["cpu_baseline"] = cpu_baseline(args, args.cpu_seconds)
    if rank == 0:
        print(json.dumps(out))
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def run_sweep(args, dev, link) -> dict:
    """The paper-shaped host-link sweeps through pinned host rings (PAPER.md:232-236
    bandwidthTest, PAPER.md:180 matrixMul): per size and direction, end-to-end GB/s of copy-engine staged (ce) and
    zero-copy (zc) serving, the faster one, and its wire bytes as a fraction of the measured copy-engine link in
    that direction (`link`, measured in this run).  workload.LinkSweep documents what one call includes."""
    import torch
    from paper_conf_sc_eilingkkflm23_b200 import gen, workload
    lo, hi = (int(x) for x in args.sweep_log2.split("-"))
    sizes = list(range(lo, hi + 1))
    sw = workload.LinkSweep(dev.index, dev, max_n=1 << max(max(sizes), 21))
    main = torch.cuda.current_stream(dev)
    points = []
    for lg in sizes:
        n = 1 << lg
        payload = torch.from_numpy(gen.c3_payload(lg)).to(dev)
        runs = min(400, max(10, -(-(1 << 30) // n)))  # >= 10 runs, ~1 GiB moved when affordable
        pt = {"log2n": lg, "bytes": n, "runs": runs}
        for direction, peak in (("h2d", link["ce_h2d_gbs"]), ("d2h", link["ce_d2h_gbs"])):
            sw.prepare(n, direction, payload)
            res = {}
            for mode in ("ce", "zc"):
                sw.run(mode, 3, main)
                ms = sw.run(mode, runs, main)
                wire = sw.slots[0].w_in if direction == "h2d" else sw.slots[0].w_out
                wg = wire * runs / ms / 1e6
                res[mode] = {"gbs": round(n * runs / ms / 1e6, 3), "wire_gbs": round(wg, 3),
                             "us_per_call": round(ms * 1e3 / runs, 2), "frac": round(wg / peak, 4),
                             "ok": sw.check(payload)}
            best = max(res, key=lambda m: res[m]["gbs"] if res[m]["ok"] else -1)
            pt[direction] = {"best": best, "gbs": res[best]["gbs"], "frac": res[best]["frac"],
                             "ok": res["ce"]["ok"] and res["zc"]["ok"], **res}
        points.append(pt)
        del payload
    cutoff = None
    for pt in reversed(points):
        if pt["h2d"]["frac"] >= 0.8 and pt["d2h"]["frac"] >= 0.8:
            cutoff = pt["bytes"]
        else:
            break
    # C2: the matrixMul batch (two HtoD CALLs, one DtoH) served as one step
    sw.prepare_c2()
    w_in, w_out = sw.slots[0].w_in, sw.slots[0].w_out
    bound_ms = max(w_in / link["ce_h2d_gbs"], w_out / link["ce_d2h_gbs"], (w_in + w_out) / link["ce_bidir_gbs"]) / 1e6
    c2 = {"payload_bytes": 2_048_000, "wire_in": w_in, "wire_out": w_out, "link_bound_us": round(bound_ms * 1e3, 2)}
    for mode in ("ce", "zc"):
        sw.run(mode, 5, main)
        ms = sw.run(mode, 200, main) / 200
        c2[mode] = {"us_per_batch": round(ms * 1e3, 2), "gbs": round(2_048_000 / ms / 1e6, 3),
                    "frac": round(bound_ms / ms, 4), "ok": sw.check(None)}
    c2["best"] = max(("ce", "zc"), key=lambda m: c2[m]["gbs"] if c2[m]["ok"] else -1)
    del sw
    torch.cuda.empty_cache()
    return {"c3": points, "c2_matrixMul": c2,
            "cutoff_bytes_frac_ge_0.8": cutoff,
            "link": {k: link[k] for k in ("ce_h2d_gbs", "ce_d2h_gbs", "ce_bidir_gbs")},
            "how": "one memcpy CALL per run (bandwidthTest), 2 calls in flight; ce = crk_ring_copy in + crk_serve from "
                   "HBM + crk_ring_copy out; zc = crk_serve on the pinned rings; each run includes the host->device "
                   "copy of its CALL and the device->host copy of its REPLY; CUDA events around all runs of a size; "
                   "frac = wire bytes in that direction / time / measured copy-engine link (C2: link-bound time / "
                   "time)"}


def shaped_link_ms(dev, n_in: int, n_out: int) -> float:
    """The copy engines alone moving exactly one step's wire bytes: n_in host->device and n_out device->host at
    the same time (pinned host memory, one copy per direction), best of 3 after a warm-up.  The e2e step moves
    the same bytes over the same link, so it cannot be faster; unlike the LP bound max(in/h2d, out/d2h,
    (in+out)/bidir) this needs no assumption about how the link shares its two directions."""
    import torch
    h, h2 = torch.empty(n_in, dtype=torch.uint8, pin_memory=True), torch.empty(n_out, dtype=torch.uint8, pin_memory=True)
    d, d2 = torch.empty(n_in, dtype=torch.uint8, device=dev), torch.empty(n_out, dtype=torch.uint8, device=dev)
    s1, s2 = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
    ts = []
    for _ in range(4):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        with torch.cuda.stream(s1):
            d.copy_(h, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)
        torch.cuda.synchronize()
        ts.append(time.perf_counter() - t0)
    del h, h2, d, d2
    return min(ts[1:]) * 1e3


def host_link_peaks(dev, nbytes: int = 512 * MiB) -> dict:
    import torch
    h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    h2 = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    d2 = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    s1, s2 = torch.cuda.Stream(dev), torch.cuda.Stream(dev)

    def best(fn, bytes_):
        ts = []
        for _ in range(4):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            fn()
            torch.cuda.synchronize()
            ts.append(time.perf_counter() - t0)
        return bytes_ / min(ts[1:]) / 1e9

    def bi():
        with torch.cuda.stream(s1):
            d.copy_(h, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)

    r = {"ce_h2d_gbs": round(best(lambda: d.copy_(h, non_blocking=True), nbytes), 2),
         "ce_d2h_gbs": round(best(lambda: h2.copy_(d2, non_blocking=True), nbytes), 2),
         "ce_bidir_gbs": round(best(bi, 2 * nbytes), 2)}
    del h, h2, d, d2
    return r


if __name__ == "__main__":
    main()
