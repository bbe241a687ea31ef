// K4 / K5 / K6 / K7: the bulk movers.
//
// Work is a list of jobs (scratch.jobs).  A DEC job gathers logical bytes [loff, loff + n) of an indexed
// record from the ring into dst (opaque unpad/scatter, K4) with an optional per-element byte swap
// (typed arrays, K5).  An ENC job writes a whole framed record (REPLY/CALL header words, XDR items from
// device memory with optional swap, zero pads, RFC 5531 §11 fragment headers) into an output ring
// (K6 / K7).  Each job's output range is cut into tiles aligned to tile_bytes in OUTPUT address space,
// so no 16-byte output chunk is shared by two tiles; tile counts are prefix-summed (K2) and persistent
// CTAs claim tiles with an atomic cursor.
//
// Inside a tile the output is a sequence of segments, each an affine map output -> source (one
// fragment of a record on decode; one fragment x one data piece on encode).  Interior 16-byte output
// chunks of a segment are built from two aligned 16-byte source loads joined by a funnel shift (the
// shift is constant per segment; the second load comes from the neighbour lane by shuffle) and
// byte-swapped per element; the at most 30 edge bytes of a segment are computed one by one with the
// exact logical -> physical map, which also covers elements split across fragments.
#include "crk_device.cuh"
#include "crk_logical.cuh"

namespace crk {

namespace {

constexpr int kU = 4;  // 16-byte chunks per lane per warp-slice iteration

struct MoveParams {
  IndexDev ix;
  Scratch sc;
  ConfigDev cfg;
  const uint64_t* prefix;  // [n_jobs + 1] exclusive tile prefix
  const uint32_t* n_jobs_dev;
  const uint64_t* total_tiles;
};

// Generic chunk loop over nch aligned output chunks.  load(i) returns source chunk i of the aligned
// source window (already element-swapped on encode); store(i, v) writes output chunk i.
template <class Load, class Store>
__device__ __forceinline__ void chunk_loop(uint64_t nch, uint32_t sh, const Load& load, const Store& store) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
  const uint4 z = make_uint4(0, 0, 0, 0);
  for (uint64_t base = (uint64_t)warp * 32 * kU; base < nch; base += (uint64_t)nwarps * 32 * kU) {
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

// ------------------------------------------------------------------------------------------- DEC
struct DecCtx {
  LogicalRecord L;
  uint64_t dst, loff;
  uint32_t es;
};

// exact source of destination byte x (element e, byte j) = logical byte loff + e*es + (es-1-j)
__device__ __forceinline__ uint8_t dec_exact_byte(DecCtx& c, uint64_t x) {
  const uint64_t i = x - c.dst;
  const uint64_t e = i / c.es, j = i - e * c.es;
  return c.L.byte(c.loff + e * c.es + (c.es - 1 - j));
}

__device__ void dec_segment(DecCtx& c, uint64_t xa, uint64_t xb, uint64_t src_at_xa) {
  const uint64_t c0 = (xa + 15) & ~15ull, c1 = xb & ~15ull;
  const RingDesc R = c.L.R;
  auto edge = [&](uint64_t ea, uint64_t eb) {
    for (uint64_t x = ea + threadIdx.x; x < eb; x += blockDim.x) {
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
  chunk_loop((c1 - c0) >> 4, sh,
             [&](uint64_t i) { return ld16_stream(R.base + ((ab + 16 * i) & R.mask)); },
             [&](uint64_t i, uint4 v) { st16(reinterpret_cast<void*>(c0 + 16 * i), swap16(v, es)); });
}

// ------------------------------------------------------------------------------------------- ENC
struct EncCtx {
  RingDesc O;
  uint64_t start;   // cursor of the record's first byte
  uint64_t Ll;      // logical length
  uint32_t F, n_lens, nfr, np;
  const uint64_t* lens;    // explicit framing: fragment lengths
  const uint64_t* wstart;  // explicit framing: fragment wire starts (exclusive prefix of len + 4)
  const Piece* P;          // smem
};
struct Frag {
  uint64_t fw, len, lf;  // wire start (rel), data length, logical start
  uint32_t last;
};
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
    uint64_t f = w / (c.F + 4);
    return (uint32_t)(f < c.nfr ? f : c.nfr - 1);
  }
  uint32_t lo = 0, hi = c.nfr;  // largest f with wstart[f] <= w
  while (hi - lo > 1) {
    uint32_t mid = (lo + hi) >> 1;
    if (c.wstart[mid] <= w) lo = mid; else hi = mid;
  }
  return lo;
}
// Byte at logical offset l of the record (l < Ll): header words, data (with swap) or zero pad.
__device__ __forceinline__ uint8_t enc_logical_byte(const EncCtx& c, uint64_t l) {
  for (uint32_t k = 0; k < c.np; ++k) {
    const Piece& p = c.P[k];
    if (p.type == PIECE_WORDS) {
      if (l < p.loff + p.nbytes) {
        const uint64_t i = l - p.loff;
        return (uint8_t)(p.words[i >> 2] >> (24 - 8 * (i & 3)));
      }
    } else {
      const uint64_t ext = p.nbytes + ((4 - (p.nbytes & 3)) & 3);
      if (l < p.loff + ext) {
        const uint64_t i = l - p.loff;
        if (i >= p.nbytes) return 0;  // RFC 4506 §3 zero pad
        const uint64_t e = i / p.esize, j = i - e * p.esize;
        return *reinterpret_cast<const uint8_t*>(p.src + e * p.esize + (p.esize - 1 - j));
      }
    }
  }
  return 0;
}
__device__ __forceinline__ void enc_put(const EncCtx& c, uint64_t w, uint8_t v) {
  c.O.base[(c.start + w) & c.O.mask] = v;
}
// per-byte output of wire range [wa, wb) inside fragment fr
__device__ void enc_bytes(const EncCtx& c, const Frag& fr, uint64_t wa, uint64_t wb) {
  for (uint64_t w = wa + threadIdx.x; w < wb; w += blockDim.x) {
    const uint64_t q = w - fr.fw;
    uint8_t v;
    if (q < 4) {
      const uint32_t h = (uint32_t)fr.len | (fr.last << 31);  // RFC 5531 §11 record mark
      v = (uint8_t)(h >> (24 - 8 * q));
    } else {
      v = enc_logical_byte(c, fr.lf + (q - 4));
    }
    enc_put(c, w, v);
  }
}
// data segment: wire [wa, wb) (inside one fragment's data, one DATA piece's payload), first source
// byte address src_at_wa in V order (element-swapped stream of the piece)
__device__ void enc_segment(const EncCtx& c, const Frag& fr, uint64_t wa, uint64_t wb, const Piece& p,
                            uint64_t l_at_wa) {
  const uint64_t ca = c.start + wa, cb = c.start + wb;  // cursors
  const uint64_t c0 = (ca + 15) & ~15ull, c1 = cb & ~15ull;
  if (c0 >= c1) { enc_bytes(c, fr, wa, wb); return; }
  enc_bytes(c, fr, wa, wa + (c0 - ca));
  enc_bytes(c, fr, wb - (cb - c1), wb);
  const uint64_t s0 = p.src + (l_at_wa - p.loff) + (c0 - ca);
  const uint32_t sh = (uint32_t)(s0 & 15), es = p.esize;
  const uint64_t ab = s0 - sh;
  const RingDesc O = c.O;
  chunk_loop((c1 - c0) >> 4, sh,
             [&](uint64_t i) { return swap16(ld16_stream(reinterpret_cast<const void*>(ab + 16 * i)), es); },
             [&](uint64_t i, uint4 v) { st16(O.base + ((c0 + 16 * i) & O.mask), v); });
}

__device__ void enc_tile(EncCtx& c, uint64_t ra, uint64_t rb) {
  uint32_t f = enc_frag_of(c, ra);
  uint64_t w = ra;
  while (w < rb) {
    const Frag fr = enc_frag(c, f);
    const uint64_t fend = fr.fw + 4 + fr.len;
    // header
    if (w < fr.fw + 4) {
      const uint64_t he = min(rb, fr.fw + 4);
      enc_bytes(c, fr, w, he);
      w = he;
    }
    // data run of this fragment inside the tile, piece by piece
    const uint64_t de = min(rb, fend);
    while (w < de) {
      const uint64_t l = fr.lf + (w - fr.fw - 4);
      // piece holding logical l
      uint32_t k = 0;
      for (; k + 1 < c.np; ++k) if (c.P[k + 1].loff > l) break;
      const Piece& p = c.P[k];
      const uint64_t pext = p.type == PIECE_WORDS ? p.nbytes : p.nbytes + ((4 - (p.nbytes & 3)) & 3);
      const uint64_t run_end_l = min(p.loff + pext, fr.lf + fr.len);
      const uint64_t run_end_w = min(de, fr.fw + 4 + (run_end_l - fr.lf));
      if (p.type == PIECE_DATA && l < p.loff + p.nbytes) {
        const uint64_t dend_l = min(p.loff + p.nbytes, fr.lf + fr.len);
        const uint64_t dend_w = min(de, fr.fw + 4 + (dend_l - fr.lf));
        enc_segment(c, fr, w, dend_w, p, l);
        enc_bytes(c, fr, dend_w, run_end_w);  // pad bytes (if in this run)
      } else {
        enc_bytes(c, fr, w, run_end_w);
      }
      w = run_end_w;
    }
    f++;
  }
}

// ------------------------------------------------------------------------------------------- kernel
__global__ void __launch_bounds__(kMoveThreads) mover_kernel(MoveParams M) {
  __shared__ Job sj;
  __shared__ __align__(16) Piece sp[kMaxPieces];
  __shared__ uint32_t s_tile, s_job, s_k0;
  __shared__ uint64_t s_pj;
  const uint64_t total = *M.total_tiles;
  const uint32_t n_jobs = *M.n_jobs_dev;
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (;;) {
    if (threadIdx.x == 0) s_tile = atomicAdd(M.sc.counters, 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    if (tile >= total) break;
    if (warp == 0) {  // 32-ary search: last job j with prefix[j] <= tile
      uint32_t lo = 0, hi = n_jobs;
      while (hi - lo > 1) {
        const uint32_t step = (hi - lo + 31) / 32;
        const uint32_t idx = lo + lane * step;
        const bool pred = idx < hi && M.prefix[idx] <= tile;
        const uint32_t m = __ballot_sync(0xffffffffu, pred);
        const uint32_t l = 31 - __clz(m);
        lo = lo + l * step;
        hi = min(hi, lo + step);
      }
      if (lane == 0) { s_job = lo; s_pj = M.prefix[lo]; }
    }
    __syncthreads();
    if (threadIdx.x < sizeof(Job) / 4)
      reinterpret_cast<uint32_t*>(&sj)[threadIdx.x] =
          reinterpret_cast<const uint32_t*>(M.sc.jobs + s_job)[threadIdx.x];
    __syncthreads();
    const uint64_t t = tile - s_pj;
    const uint32_t shf = M.cfg.tile_shift;
    const uint64_t A = sj.out_start >> shf;
    const uint64_t a = max(sj.out_start, (A + t) << shf), b = min(sj.out_end, (A + t + 1) << shf);
    if (sj.type == JOB_DEC) {
      DecCtx c;
      const uint32_t rec = sj.rec;
      const uint32_t slot = M.ix.p_slot[rec];
      c.L.init(M.ix, M.ix.rings[M.ix.p_ring[rec]], slot);
      c.dst = sj.out_start;
      c.loff = sj.loff;
      c.es = sj.esize;
      if (threadIdx.x == 0) s_k0 = c.L.find(c.loff + (a - c.dst));
      __syncthreads();
      uint32_t k = s_k0;
      c.L.hint = k;
      uint64_t r = a;
      while (r < b && k < c.L.nfrags) {
        const uint64_t ls = c.L.lstart[k], fl = c.L.flen(k), ph = c.L.phys[k];
        const uint64_t fend = c.dst + (ls + fl - c.loff);
        const uint64_t sb = min(b, fend);
        if (sb > r) {
          dec_segment(c, r, sb, ph + (c.loff + (r - c.dst) - ls));
          r = sb;
        }
        ++k;
      }
    } else if (sj.type == JOB_ENC) {
      for (uint32_t i = threadIdx.x; i < sj.n_pieces * (sizeof(Piece) / 4); i += blockDim.x)
        reinterpret_cast<uint32_t*>(sp)[i] = reinterpret_cast<const uint32_t*>(M.sc.pieces + sj.piece0)[i];
      __syncthreads();
      EncCtx c;
      c.O = M.sc.out_rings[sj.out_ring];
      c.start = sj.out_start;
      c.Ll = sj.loff;
      c.F = sj.F;
      c.n_lens = sj.n_lens;
      c.np = sj.n_pieces;
      c.P = sp;
      c.lens = M.sc.lens_pool + sj.lens0;
      c.wstart = M.sc.lens_pool + M.sc.max_lens + sj.lens0;
      c.nfr = c.F ? (uint32_t)(c.Ll == 0 ? 1 : (c.Ll + c.F - 1) / c.F) : c.n_lens;
      enc_tile(c, a - c.start, b - c.start);
    }
    __syncthreads();
  }
}

// tiles per job: output range cut at tile_bytes-aligned boundaries
__global__ void plan_count_kernel(Scratch sc, ConfigDev cfg, uint64_t* tiles, const uint32_t* n_jobs_dev) {
  const uint32_t n = *n_jobs_dev;
  if (blockIdx.x == 0 && threadIdx.x == 0) sc.counters[0] = 0;  // mover tile cursor
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n; j += gridDim.x * blockDim.x) {
    const Job jb = sc.jobs[j];
    uint64_t c = 0;
    if (jb.type != JOB_NONE && jb.out_end > jb.out_start)
      c = ((jb.out_end - 1) >> cfg.tile_shift) - (jb.out_start >> cfg.tile_shift) + 1;
    tiles[j] = c;
  }
}

}  // namespace

cudaError_t launch_plan_and_move(const IndexDev* ix, const ConfigDev& cfg, Scratch& sc, uint32_t max_jobs_bound,
                                 int sms, int move_ctas, cudaStream_t s) {
  uint64_t* tiles = sc.scan_tmp;  // [max_jobs + 1]
  uint64_t* total = sc.scan_tmp + sc.max_jobs + 1;
  const uint32_t* n_jobs_dev = sc.counters + 1;
  const uint32_t cnt_blocks = max_jobs_bound ? (max_jobs_bound + 255) / 256 : 1;
  plan_count_kernel<<<min(cnt_blocks, (uint32_t)sms * 8), 256, 0, s>>>(sc, cfg, tiles, n_jobs_dev);
  count_launch();
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  e = launch_exclusive_scan_u64(tiles, max_jobs_bound, n_jobs_dev, total, sc, s);
  if (e != cudaSuccess) return e;
  MoveParams M;
  if (ix) M.ix = *ix; else memset(&M.ix, 0, sizeof(M.ix));
  M.sc = sc;
  M.cfg = cfg;
  M.prefix = tiles;
  M.n_jobs_dev = n_jobs_dev;
  M.total_tiles = total;
  prof_mark(PROF_MOVE, true, s);
  mover_kernel<<<move_ctas, kMoveThreads, 0, s>>>(M);
  count_launch();
  prof_mark(PROF_MOVE, false, s);
  return cudaGetLastError();
}

int mover_occupancy() {
  int n = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, mover_kernel, kMoveThreads, 0);
  return n;
}

}  // namespace crk
