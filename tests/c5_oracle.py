"""The oracle's side of a C5 endpoint: gen's seeded descriptions encoded with the
oracle's own encoder (oracle.encode_call), and the region as it stands before a serve (DtoH sources in place).
Test infrastructure only; shares nothing with the CUDA path except gen's draws."""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import gen

MiB = 1 << 20


@dataclass
class OracleEndpoint:
    cfg: O.Config
    streams: list
    region: np.ndarray   # initial region: DtoH sources placed, HtoD destinations zero
    wires: list          # per stream: the ring bytes [0, tail) as uint8 arrays

    def ring_array(self, i: int, cap: int) -> np.ndarray:
        r = np.zeros(cap, np.uint8)
        r[:len(self.wires[i])] = self.wires[i]
        return r


def oracle_endpoint(rank: int, n_streams: int, region_bytes: int, base: int, payload_per_stream: int = 64 * MiB,
                    h2d_frac: float = 0.5, F: int = 65536) -> OracleEndpoint:
    """Same draws as workload.c5_endpoint (budget rule included); `base` = the device region's address, which
    the CALLs carry as their pointers."""
    budget = payload_per_stream if h2d_frac >= 1.0 else payload_per_stream - payload_per_stream // 16
    streams, rb = gen.c5_endpoint(rank, n_streams=n_streams, payload_per_stream=payload_per_stream,
                                  h2d_budget=budget, h2d_frac=h2d_frac)
    assert rb == region_bytes, (rb, region_bytes)
    return oracle_endpoint_of(streams, region_bytes, base, F)


def oracle_endpoint_of(streams: list, region_bytes: int, base: int, F: int = 65536) -> OracleEndpoint:
    """The oracle's encoding of any gen memcpy streams (C5, the NEXT-2 profiles)."""
    cfg = O.Config(prog=gen.PROG, vers=gen.VERS, proc_h2d=gen.PROC_H2D, proc_d2h=gen.PROC_D2H, frag_payload=F)
    region = np.zeros(region_bytes + 256, np.uint8)
    wires = []
    for s in streams:
        parts = []
        for r in s.records:
            d = gen.random_bytes(r.seed & 0xFFFFFFFF, r.size)
            if r.kind == gen.PROC_H2D:
                parts.append(O.encode_call(r.xid, r.kind, [(O.K_U64, base + r.region_off), (O.K_OPAQUE_VAR, d),
                                                           (O.K_U64, r.size)], cfg))
            else:
                region[r.region_off:r.region_off + r.size] = d
                parts.append(O.encode_call(r.xid, r.kind, [(O.K_U64, base + r.region_off), (O.K_U64, r.size)], cfg))
        wires.append(np.frombuffer(b"".join(parts), np.uint8))
    return OracleEndpoint(cfg, streams, region, wires)
