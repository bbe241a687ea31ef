// Generic (non-staged) movers: decode of a logical-record range into dst and encode of a framed record's
// wire range, done by a team of warps with direct 16-byte loads and warp-shuffle realignment.  Used by the
// mover kernel's fallback path (k_move.cu) and by the persistent server (k_server.cu).
#pragma once
#include "crk_device.cuh"
#include "crk_logical.cuh"

namespace crk {

namespace {

constexpr int kU = 4;           // 16-byte chunks per lane per warp-slice iteration (generic path)
enum : uint32_t { SEG_DATA = 0, SEG_LIT = 1 };


struct Team {              // the threads that move one tile / job
  uint32_t tid, nthr, warp, nwarps;
};

// ------------------------------------------------------------------------------------------- generic path
// Chunk loop over nch aligned output chunks with direct global loads: load(i) returns source chunk i of
// the aligned source window; the second chunk of the funnel comes from the neighbour lane.
template <class Load, class Store>
__device__ __forceinline__ void chunk_loop(const Team& T, uint64_t nch, uint32_t sh, const Load& load,
                                           const Store& store) {
  const uint32_t lane = threadIdx.x & 31;
  const uint4 z = make_uint4(0, 0, 0, 0);
  for (uint64_t base = (uint64_t)T.warp * 32 * kU; base < nch; base += (uint64_t)T.nwarps * 32 * kU) {
    uint4 A[kU];
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      const uint64_t i = base + u * 32 + lane;
      A[u] = i < nch ? load(i) : z;
    }
    if (sh == 0) {
#pragma unroll
      for (int u = 0; u < kU; ++u) {
        const uint64_t i = base + u * 32 + lane;
        if (i < nch) store(i, A[u]);
      }
      continue;
    }
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      uint4 B;
      B.x = __shfl_down_sync(0xffffffffu, A[u].x, 1);
      B.y = __shfl_down_sync(0xffffffffu, A[u].y, 1);
      B.z = __shfl_down_sync(0xffffffffu, A[u].z, 1);
      B.w = __shfl_down_sync(0xffffffffu, A[u].w, 1);
      uint4 Bn = z;
      if (u + 1 < kU) {
        Bn.x = __shfl_sync(0xffffffffu, A[u + 1].x, 0);
        Bn.y = __shfl_sync(0xffffffffu, A[u + 1].y, 0);
        Bn.z = __shfl_sync(0xffffffffu, A[u + 1].z, 0);
        Bn.w = __shfl_sync(0xffffffffu, A[u + 1].w, 0);
      }
      const uint64_t i = base + u * 32 + lane;
      if (i < nch) {
        if (lane == 31) B = (u + 1 < kU && i + 1 < nch) ? Bn : load(i + 1);
        else if (i + 1 >= nch) B = load(i + 1);
        store(i, funnel16(A[u], B, sh));
      }
    }
  }
}

// ---- DEC
struct DecCtx {
  LogicalRecord L;
  uint64_t dst, loff;
  uint32_t es;
};
// From the decode job's own record coordinates (dec_job: first fragment, count, ring, first fragment's length):
// one round trip for the ring descriptor instead of the job -> record -> fragment table chain.
__device__ __forceinline__ void dec_ctx_init(DecCtx& c, const IndexDev& ix, const Job& j, const RingDesc& R) {
  LogicalRecord& L = c.L;
  L.R = R;
  L.frag0 = j.piece0;
  L.nfrags = j.n_pieces;
  L.len = ~0ull;  // not needed by the decode paths (they stay inside the job's range)
  L.phys = ix.frag_phys + j.piece0;
  L.lstart = ix.frag_lstart + j.piece0;
  L.hdr = ix.frag_hdr + j.piece0;
  L.hint = 0;
  L.F0 = j.F;
  c.dst = j.out_start;
  c.loff = j.loff;
  c.es = j.esize;
}
__device__ __forceinline__ void dec_ctx_init(DecCtx& c, const IndexDev& ix, const Job& j) {
  dec_ctx_init(c, ix, j, ix.rings[j.out_ring]);
}
// exact source of destination byte x (element e, byte j) = logical byte loff + e*es + (es-1-j)
__device__ __forceinline__ uint8_t dec_exact_byte(DecCtx& c, uint64_t x) {
  const uint64_t i = x - c.dst;
  const uint64_t e = i / c.es, j = i - e * c.es;
  return c.L.byte(c.loff + e * c.es + (c.es - 1 - j));
}
__device__ void dec_segment_direct(const Team& T, DecCtx& c, uint64_t xa, uint64_t xb, uint64_t src_at_xa) {
  const uint64_t c0 = (xa + 15) & ~15ull, c1 = xb & ~15ull;
  const RingDesc R = c.L.R;
  auto edge = [&](uint64_t ea, uint64_t eb) {
    for (uint64_t x = ea + T.tid; x < eb; x += T.nthr) {
      const uint8_t v = c.es == 1 ? ring_byte(R, src_at_xa + (x - xa)) : dec_exact_byte(c, x);
      *reinterpret_cast<uint8_t*>(x) = v;
    }
  };
  if (c0 >= c1) { edge(xa, xb); return; }
  edge(xa, c0);
  edge(c1, xb);
  const uint64_t s0 = src_at_xa + (c0 - xa);
  const uint32_t sh = (uint32_t)(s0 & 15);
  const uint64_t ab = s0 - sh;
  const uint32_t es = c.es;
  chunk_loop(T, (c1 - c0) >> 4, sh, [&](uint64_t i) { return ld16_stream(R.base + ((ab + 16 * i) & R.mask)); },
             [&](uint64_t i, uint4 v) { st16(reinterpret_cast<void*>(c0 + 16 * i), swap16(v, es)); });
}
__device__ void dec_tile_generic(const Team& T, DecCtx& c, uint64_t a, uint64_t b, uint32_t k) {
  c.L.hint = k;
  uint64_t r = a;
  while (r < b && k < c.L.nfrags) {
    const uint64_t ls = c.L.lstart[k], fl = c.L.flen(k), ph = c.L.phys[k];
    const uint64_t sb = min(b, c.dst + (ls + fl - c.loff));
    if (sb > r) {
      dec_segment_direct(T, c, r, sb, ph + (c.loff + (r - c.dst) - ls));
      r = sb;
    }
    ++k;
  }
}

// ---- ENC
struct EncCtx {
  RingDesc O;
  uint64_t start;   // cursor of the record's first byte
  uint64_t Ll;      // logical length
  uint32_t F, nfr, np;
  const uint64_t* lens;    // explicit framing: fragment lengths
  const uint64_t* wstart;  // explicit framing: fragment wire starts (exclusive prefix of len + 4)
  const Piece* P;
};
struct Frag {
  uint64_t fw, len, lf;  // wire start (rel), data length, logical start
  uint32_t last;
};
__device__ __forceinline__ void enc_ctx_init(EncCtx& c, const Scratch& sc, const Job& j, const RingDesc& O,
                                             const Piece* P) {
  c.O = O;
  c.start = j.out_start;
  c.Ll = j.loff;
  c.F = j.F;
  c.np = j.n_pieces;
  c.P = P;
  c.lens = sc.lens_pool + j.lens0;
  c.wstart = sc.lens_pool + sc.max_lens + j.lens0;
  c.nfr = c.F ? (uint32_t)(c.Ll == 0 ? 1 : (c.Ll + c.F - 1) / c.F) : j.n_lens;
}
__device__ __forceinline__ Frag enc_frag(const EncCtx& c, uint32_t f) {
  Frag r;
  if (c.F) {
    r.fw = (uint64_t)f * (c.F + 4);
    r.lf = (uint64_t)f * c.F;
    r.len = f + 1 < c.nfr ? c.F : c.Ll - r.lf;
  } else {
    r.fw = c.wstart[f];
    r.len = c.lens[f];
    r.lf = r.fw - 4ull * f;
  }
  r.last = f + 1 == c.nfr;
  return r;
}
__device__ __forceinline__ uint32_t enc_frag_of(const EncCtx& c, uint64_t w) {
  if (c.F) {
    const uint64_t f = w / (c.F + 4);
    return (uint32_t)(f < c.nfr ? f : c.nfr - 1);
  }
  uint32_t lo = 0, hi = c.nfr;  // largest f with wstart[f] <= w
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (c.wstart[mid] <= w) lo = mid; else hi = mid;
  }
  return lo;
}
__device__ __forceinline__ uint64_t piece_extent(const Piece& p) {
  return p.type == PIECE_WORDS ? p.nbytes : p.nbytes + ((4 - (p.nbytes & 3)) & 3);
}
// Byte at logical offset l of the record (l < Ll): header words, data (with swap) or zero pad.
__device__ __forceinline__ uint8_t enc_logical_byte(const EncCtx& c, uint64_t l) {
  for (uint32_t k = 0; k < c.np; ++k) {
    const Piece& p = c.P[k];
    if (l < p.loff + piece_extent(p)) {
      const uint64_t i = l - p.loff;
      if (p.type == PIECE_WORDS) return (uint8_t)(p.words[i >> 2] >> (24 - 8 * (i & 3)));
      if (i >= p.nbytes) return 0;  // RFC 4506 §3 zero pad
      const uint64_t e = i / p.esize, j = i - e * p.esize;
      return *reinterpret_cast<const uint8_t*>(p.src + e * p.esize + (p.esize - 1 - j));
    }
  }
  return 0;
}
// Wire byte w (relative to the record start): RFC 5531 §11 record mark or logical byte.
__device__ __forceinline__ uint8_t enc_wire_byte(const EncCtx& c, uint64_t w) {
  const Frag fr = enc_frag(c, enc_frag_of(c, w));
  const uint64_t q = w - fr.fw;
  if (q < 4) {
    const uint32_t h = (uint32_t)fr.len | (fr.last << 31);
    return (uint8_t)(h >> (24 - 8 * q));
  }
  return enc_logical_byte(c, fr.lf + (q - 4));
}
__device__ __forceinline__ void enc_bytes(const Team& T, const EncCtx& c, uint64_t wa, uint64_t wb) {
  for (uint64_t w = wa + T.tid; w < wb; w += T.nthr) c.O.base[(c.start + w) & c.O.mask] = enc_wire_byte(c, w);
}
// The interior 16-byte chunks of data run [wa, wb) (the aligned chunks it covers whole), from direct loads.
__device__ void enc_segment_interior(const Team& T, const EncCtx& c, uint64_t wa, uint64_t wb, uint64_t src_at_wa,
                                     uint32_t es) {
  const uint64_t ca = c.start + wa, cb = c.start + wb;
  const uint64_t c0 = (ca + 15) & ~15ull, c1 = cb & ~15ull;
  if (c0 >= c1) return;
  const uint64_t s0 = src_at_wa + (c0 - ca);
  const uint32_t sh = (uint32_t)(s0 & 15);
  const uint64_t ab = s0 - sh;
  const RingDesc O = c.O;
  chunk_loop(T, (c1 - c0) >> 4, sh,
             [&](uint64_t i) { return swap16(ld16_stream(reinterpret_cast<const void*>(ab + 16 * i)), es); },
             [&](uint64_t i, uint4 v) { st16(O.base + ((c0 + 16 * i) & O.mask), v); });
}
__device__ void enc_segment_direct(const Team& T, const EncCtx& c, uint64_t wa, uint64_t wb, uint64_t src_at_wa,
                                   uint32_t es) {
  const uint64_t ca = c.start + wa, cb = c.start + wb;
  const uint64_t c0 = (ca + 15) & ~15ull, c1 = cb & ~15ull;
  if (c0 >= c1) { enc_bytes(T, c, wa, wb); return; }
  enc_bytes(T, c, wa, wa + (c0 - ca));
  enc_bytes(T, c, wb - (cb - c1), wb);
  enc_segment_interior(T, c, wa, wb, src_at_wa, es);
}
// The output bytes of aligned chunks [g0, g1) (absolute out-ring cursors, 16-byte aligned) that lie inside
// [xa, xb), composed chunk by chunk in registers from the exact wire map (fragment headers, REPLY / CALL words,
// pads, data edges): one 16-byte store per chunk inside [xa, xb); byte stores only for a chunk the range cuts
// (the first / last chunk of a job, shared with the neighbouring record).  Used for everything of an encode
// tile outside its data runs' interior chunks, so a send ring in pinned host memory receives whole-chunk
// writes over PCIe instead of single-byte ones (SURVEY.md §7 "PCIe efficiency").
// A warp takes two chunks at a time: lane l computes byte l & 15 of chunk l >> 4 (all 32 in parallel), the
// bytes are gathered into words and the words into the chunk's first lane with shuffles.
__device__ void enc_gap_chunks(const Team& T, const EncCtx& c, uint64_t g0, uint64_t g1, uint64_t xa, uint64_t xb) {
  const uint32_t lane = threadIdx.x & 31, j = lane & 15;
  for (uint64_t p = g0 + 32ull * T.warp; p < g1; p += 32ull * T.nwarps) {  // warp-uniform
    const uint64_t x0 = p + 16 * (lane >> 4), x = x0 + j;
    const bool in = x0 < g1 && x >= xa && x < xb;
    const bool whole = x0 < g1 && x0 >= xa && x0 + 16 <= xb;
    const uint32_t b = in ? enc_wire_byte(c, x - c.start) : 0u;
    uint32_t w = b | (__shfl_down_sync(0xffffffffu, b, 1) << 8) | (__shfl_down_sync(0xffffffffu, b, 2) << 16) |
                 (__shfl_down_sync(0xffffffffu, b, 3) << 24);  // valid at j % 4 == 0
    const uint32_t w1 = __shfl_down_sync(0xffffffffu, w, 4), w2 = __shfl_down_sync(0xffffffffu, w, 8),
                   w3 = __shfl_down_sync(0xffffffffu, w, 12);
    if (whole) {
      if (j == 0) st16(c.O.base + (x0 & c.O.mask), make_uint4(w, w1, w2, w3));
    } else if (in) {
      c.O.base[x & c.O.mask] = (uint8_t)b;
    }
  }
}
// Walks wire range [ra, rb) of the record as runs: fragment headers, then per fragment the pieces'
// data / literal parts.  emit(kind, wa, wb, src_at_wa, es) is called for each run in order.
template <class Emit>
__device__ __forceinline__ bool enc_runs(const EncCtx& c, uint64_t ra, uint64_t rb, const Emit& emit) {
  uint32_t f = enc_frag_of(c, ra);
  uint64_t w = ra;
  while (w < rb) {
    const Frag fr = enc_frag(c, f);
    const uint64_t he = min(rb, fr.fw + 4), de = min(rb, fr.fw + 4 + fr.len);
    if (w < he) {
      if (!emit(SEG_LIT, w, he, 0ull, 1u)) return false;
      w = he;
    }
    while (w < de) {
      const uint64_t l = fr.lf + (w - fr.fw - 4);
      uint32_t k = 0;
      for (; k + 1 < c.np; ++k)
        if (c.P[k + 1].loff > l) break;
      const Piece& p = c.P[k];
      const uint64_t run_end_l = min(p.loff + piece_extent(p), fr.lf + fr.len);
      const uint64_t run_end_w = min(de, fr.fw + 4 + (run_end_l - fr.lf));
      if (p.type == PIECE_DATA && l < p.loff + p.nbytes) {
        const uint64_t dend_l = min(p.loff + p.nbytes, fr.lf + fr.len);
        const uint64_t dend_w = min(de, fr.fw + 4 + (dend_l - fr.lf));
        if (!emit(SEG_DATA, w, dend_w, p.src + (l - p.loff), p.esize)) return false;
        if (dend_w < run_end_w && !emit(SEG_LIT, dend_w, run_end_w, 0ull, 1u)) return false;
      } else {
        if (!emit(SEG_LIT, w, run_end_w, 0ull, 1u)) return false;
      }
      w = run_end_w;
    }
    f++;
  }
  return true;
}
// Encode of wire range [ra, rb): each data run's interior chunks by 16-byte copies, everything between them
// (headers, words, pads, data edges) by enc_gap_chunks, in wire order.
__device__ void enc_tile_generic(const Team& T, const EncCtx& c, uint64_t ra, uint64_t rb) {
  const uint64_t xa = c.start + ra, xb = c.start + rb;
  uint64_t gap = xa & ~15ull;  // first chunk not yet written
  enc_runs(c, ra, rb, [&](uint32_t kind, uint64_t wa, uint64_t wb, uint64_t src, uint32_t es) {
    if (kind == SEG_LIT) return true;
    const uint64_t c0 = (c.start + wa + 15) & ~15ull, c1 = (c.start + wb) & ~15ull;
    if (c0 >= c1) return true;
    enc_gap_chunks(T, c, gap, c0, xa, xb);
    enc_segment_interior(T, c, wa, wb, src, es);
    gap = c1;
    return true;
  });
  enc_gap_chunks(T, c, gap, (xb + 15) & ~15ull, xa, xb);
}


}  // namespace
}  // namespace crk
