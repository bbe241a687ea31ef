// K4 / K5 / K6 / K7: the bulk movers.
//
// Work is a list of jobs (scratch.jobs).  A DEC job gathers logical bytes [loff, loff + n) of an indexed
// record from its ring into dst (opaque unpad/scatter, K4) with an optional per-element byte swap
// (typed arrays, K5).  An ENC job writes a whole framed record (REPLY/CALL header words, XDR items from
// device memory with optional swap, zero pads, RFC 5531 §11 fragment headers) into an output ring
// (K6 / K7).  Each job's output range is cut into tiles aligned to tile_bytes in OUTPUT address space,
// so no 16-byte output chunk is shared by two tiles; tile counts are prefix-summed (K2).
//
// The mover is a persistent, warp-specialised TMA pipeline.  Warp 0 (producer) claims tiles with an
// atomic cursor, resolves tile -> job -> fragments, splits the tile into segments (each an affine map
// output -> source: one fragment of a record on decode; fragment x data piece, or a literal run of
// headers / words / pad, on encode) and issues cp.async.bulk copies of every data segment's 16-byte
// aligned source window into a shared-memory stage, completing on the stage's mbarrier.  Warps 1-8
// (consumers) wait on the stage, build each aligned 16-byte output chunk from two shared-memory chunks
// with a funnel shift (constant per segment) and a per-element byte swap, store it with STG.128, and
// release the stage.  The few edge bytes of a segment (at most 30) are computed one by one from the
// exact logical -> physical map, which also covers elements split across fragments.  Tiles with more
// segments than a stage describes (fragments smaller than ~tile/8) run the generic path: the same
// segment walk done by the consumers with direct 16-byte global loads and warp-shuffle realignment.
// Two tile queues (decode jobs, encode jobs) are claimed alternately so a serve step keeps both PCIe
// directions busy when the rings live in host memory.
#include <mutex>

#include "k_move.cuh"

namespace crk {

namespace {

constexpr int kMaxSeg = 8;      // segments a stage can describe
constexpr int kMaxStages = 8;   // pipeline depth limit (runtime: cfg.stages)
#ifndef CRK_MOVER_CONSUMERS
#define CRK_MOVER_CONSUMERS 8
#endif
constexpr int kConsumerWarps = CRK_MOVER_CONSUMERS;
constexpr int kMoverThreads = 32 * (1 + kConsumerWarps);

struct Seg {               // 32 bytes
  uint64_t out_a, out_b;   // output range (DEC: dst addresses; ENC: out-ring cursors)
  uint64_t src;            // DEC: ring cursor of the byte for out_a; ENC: V-order address of the byte for out_a
  uint32_t smem_off;       // offset in the stage buffer of the aligned source window (staged only)
  uint32_t flags;          // bit 0 staged, bit 1 edge bytes staged too, bits 8-15 kind, bits 16-23 element size
};

struct StageHdr {
  uint32_t type, fallback, nseg, k0;
  uint64_t a, b;
  Job job;
  RingDesc R;              // DEC: the record's ring; ENC: the output ring
  Seg seg[kMaxSeg];
  Piece pieces[kMaxPieces];
};

struct MoveParams {
  IndexDev ix;
  Scratch sc;
  ConfigDev cfg;
  const uint64_t* prefix;  // [n_jobs] exclusive tile prefix
  const uint32_t* n_jobs_dev;
  const uint64_t* total_tiles;
  uint32_t stage_bytes;    // bytes of one stage buffer (after its header)
  uint32_t seq;            // this launch's number (launch stamp)
  uint32_t use_map;        // a run_map_kernel ran for this launch (counters[13] says whether its map applies)
  uint32_t opp_from;       // CTAs >= opp_from are opportunistic (crk_config.mover_reserve_ctas)
};

__device__ __forceinline__ uint32_t gtimer32() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return (uint32_t)t;
}
// Opportunistic CTAs (the last cfg.reserve of the grid) join only a launch that found the GPU free: the
// whole grid starts within a few microseconds of CTA 0.  When this mover launches while another batch's
// mover still holds the SMs (a pipelined server loop), its last CTAs are dispatched only when that mover
// retires, long after CTA 0 started; they exit at once, so their slots stay free for the next batch's scan /
// parse / plan kernels.  CTA 0 stamps the launch (sequence, start time) in the context's counters.
constexpr uint32_t kOppLateNs = 10000;
__device__ bool mover_cta_runs(const MoveParams& M) {
  __shared__ uint32_t go;
  volatile uint32_t* c = M.sc.counters;
  if (threadIdx.x == 0) {
    const uint32_t t = gtimer32();
    uint32_t g = 1;
    if (blockIdx.x == 0) {
      c[9] = t;
      __threadfence();
      c[8] = M.seq;
    } else if (blockIdx.x >= M.opp_from) {
      while (c[8] != M.seq && gtimer32() - t < 2 * kOppLateNs) __nanosleep(256);
      if (c[8] == M.seq) {
        __threadfence();
        g = (int32_t)(t - c[9]) < (int32_t)kOppLateNs;  // signed: a CTA that read the timer before CTA 0
                                                        // stamped it started with the launch
      }
    }
    go = g;
  }
  __syncthreads();
  return go != 0;
}

// PTX helpers (mbarrier, cp.async.bulk): crk_device.cuh
__device__ __forceinline__ uint4 lds16(const uint8_t* p) { return *reinterpret_cast<const uint4*>(p); }

// ------------------------------------------------------------------------------------------- staged path
// Interior chunks [c0, c1) of a staged data segment.  `o0` = offset in `buf` of the source byte that
// lands on output chunk c0; the chunk's bytes are buf[o0 + 16 i .. + 16).
__device__ __forceinline__ void staged_chunks(const Team& T, const uint8_t* buf, uint32_t o0, uint64_t nch,
                                              uint64_t out0, const RingDesc* O, uint32_t es, bool dec) {
  const uint32_t r = o0 & 15;
  const uint8_t* q0 = buf + (o0 & ~15u);
  for (uint64_t i = T.tid; i < nch; i += T.nthr) {
    uint4 lo = lds16(q0 + 16 * i), v;
    if (dec) {
      v = r ? funnel16(lo, lds16(q0 + 16 * i + 16), r) : lo;
      v = swap16(v, es);
      st16(reinterpret_cast<void*>(out0 + 16 * i), v);
    } else {
      lo = swap16(lo, es);
      v = r ? funnel16(lo, swap16(lds16(q0 + 16 * i + 16), es), r) : lo;
      st16(O->base + ((out0 + 16 * i) & O->mask), v);
    }
  }
}


// ------------------------------------------------------------------------------------------- producer state
constexpr uint32_t kWin = 64;  // fragment entries cached per producer
struct ProdCache {
  Job job;
  Piece pieces[kMaxPieces];
  RingDesc R;                 // DEC: the record's ring; ENC: the output ring
  uint64_t rec_len, F0;
  uint32_t frag0, nfrags;     // absolute index of the record's first fragment, fragment count
  uint32_t wk0, wn;           // window: fragments [wk0, wk0 + wn) of the record
  uint32_t hint;
  uint64_t lstart[kWin], phys[kWin];
  uint32_t hdr[kWin];
};

// Loads job j (and its pieces / ring / record) into the producer cache; the whole warp calls it.
__device__ __forceinline__ void producer_load_job(ProdCache& pc, const MoveParams& M, uint32_t j, uint32_t lane,
                                                  const RingDesc* ring_s) {
  if (lane < sizeof(Job) / 4)
    reinterpret_cast<uint32_t*>(&pc.job)[lane] = reinterpret_cast<const uint32_t*>(M.sc.jobs + j)[lane];
  __syncwarp();
  const Job& J = pc.job;
  if (J.type == JOB_ENC) {
    for (uint32_t i = lane; i < J.n_pieces * (sizeof(Piece) / 4); i += 32)
      reinterpret_cast<uint32_t*>(pc.pieces)[i] = reinterpret_cast<const uint32_t*>(M.sc.pieces + J.piece0)[i];
    if (lane == 0) pc.R = M.sc.out_rings[J.out_ring];
  } else if (J.type == JOB_DEC && lane == 0) {  // the record's coordinates travel in the job (dec_job)
    pc.R = ring_s[J.out_ring];
    pc.frag0 = J.piece0;
    pc.nfrags = J.n_pieces;
    pc.F0 = J.F;
    pc.wn = 0;
    pc.hint = 0;
  }
  __syncwarp();
}

__device__ __forceinline__ void producer_frag(const ProdCache& pc, const MoveParams& M, uint32_t k, uint64_t& ls,
                                              uint64_t& ph, uint32_t& hd) {
  if (k >= pc.wk0 && k < pc.wk0 + pc.wn) {
    const uint32_t i = k - pc.wk0;
    ls = pc.lstart[i]; ph = pc.phys[i]; hd = pc.hdr[i];
  } else {
    const uint64_t g = (uint64_t)pc.frag0 + k;
    ls = M.ix.frag_lstart[g]; ph = M.ix.frag_phys[g]; hd = M.ix.frag_hdr[g];
  }
}

// Fragment holding logical offset `off` of the current record; makes sure the window covers it and
// the next kMaxSeg fragments.  The whole warp calls it; lane 0's answer is returned to every lane.
__device__ uint32_t producer_frag_window(ProdCache& pc, const MoveParams& M, uint64_t off, uint32_t lane) {
  uint32_t k0 = 0;
  if (pc.wn == 0 && pc.F0) {
    // fresh job: fill the window around the uniform-stride guess in one round trip, so the search below
    // runs from shared memory (greedy F framing puts offset off in fragment off / F0 exactly)
    const uint32_t n = pc.nfrags;
    const uint64_t gs = off / pc.F0;
    const uint32_t g = gs < n ? (uint32_t)gs : n - 1;
    const uint32_t base = g > 0 ? g - 1 : 0, cnt = min(kWin, n - base);
    for (uint32_t i = lane; i < cnt; i += 32) {
      const uint64_t q = (uint64_t)pc.frag0 + base + i;
      pc.lstart[i] = M.ix.frag_lstart[q];
      pc.phys[i] = M.ix.frag_phys[q];
      pc.hdr[i] = M.ix.frag_hdr[q];
    }
    __syncwarp();
    if (lane == 0) { pc.wk0 = base; pc.wn = cnt; pc.hint = g; }
    __syncwarp();
  }
  if (lane == 0) {
    auto holds = [&](uint32_t k) {
      uint64_t ls, ph;
      uint32_t hd;
      producer_frag(pc, M, k, ls, ph, hd);
      return off >= ls && off < ls + (hd & 0x7fffffffu);
    };
    const uint32_t n = pc.nfrags;
    uint32_t k = pc.hint;
    bool found = k < n && holds(k);
    for (uint32_t i = 1; !found && i <= 2 && k + i < n; ++i)
      if (holds(k + i)) { k += i; found = true; }
    if (!found && pc.F0) {
      const uint64_t g = off / pc.F0;
      if (g < n && holds((uint32_t)g)) { k = (uint32_t)g; found = true; }
    }
    if (!found) {  // binary search over the record's fragments: largest k with lstart[k] <= off
      uint32_t lo = 0, hi = n;
      while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        uint64_t ls, ph;
        uint32_t hd;
        producer_frag(pc, M, mid, ls, ph, hd);
        if (ls <= off) lo = mid; else hi = mid;
      }
      k = lo;
    }
    pc.hint = k;
    k0 = k;
  }
  k0 = __shfl_sync(0xffffffffu, k0, 0);
  const uint32_t n = pc.nfrags;
  const uint32_t want_end = min(n, k0 + kMaxSeg + 1);
  if (!(k0 >= pc.wk0 && want_end <= pc.wk0 + pc.wn)) {
    __syncwarp();
    const uint32_t base = k0, cnt = min(kWin, n - base);
    for (uint32_t i = lane; i < cnt; i += 32) {
      const uint64_t g = (uint64_t)pc.frag0 + base + i;
      pc.lstart[i] = M.ix.frag_lstart[g];
      pc.phys[i] = M.ix.frag_phys[g];
      pc.hdr[i] = M.ix.frag_hdr[g];
    }
    if (lane == 0) { pc.wk0 = base; pc.wn = cnt; }
    __syncwarp();
  }
  return k0;
}

// ------------------------------------------------------------------------------------------- kernel
__device__ __forceinline__ uint32_t find_job(const uint64_t* prefix, uint32_t n_jobs, uint64_t tile, uint32_t lane) {
  uint32_t lo = 0, hi = n_jobs;  // last j with prefix[j] <= tile (32-ary search, one warp)
  while (hi - lo > 1) {
    const uint32_t step = (hi - lo + 31) / 32;
    const uint32_t idx = lo + lane * step;
    const bool pred = idx < hi && prefix[idx] <= tile;
    const uint32_t m = __ballot_sync(0xffffffffu, pred);
    lo = lo + (31 - __clz(m)) * step;
    hi = min(hi, lo + step);
  }
  return lo;
}

#ifndef CRK_MOVER_MIN_BLOCKS
#define CRK_MOVER_MIN_BLOCKS 2
#endif
__global__ void __launch_bounds__(kMoverThreads, CRK_MOVER_MIN_BLOCKS) mover_kernel(MoveParams M) {
  pdl_entry();
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ __align__(8) uint64_t full[kMaxStages], empty[kMaxStages];
  const uint32_t kStages = M.cfg.stages;
  const uint32_t stage_stride = (sizeof(StageHdr) + 127) / 128 * 128 + M.stage_bytes;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (!mover_cta_runs(M)) return;
  TL_BEGIN(M.cfg, TL_MOVE);
  if (threadIdx.x == 0) {
    for (uint32_t s = 0; s < kStages; ++s) {
      mbar_init(&full[s], 32);  // every producer lane arrives after its own writes to the stage
      mbar_init(&empty[s], 32 * kConsumerWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const uint64_t total = *M.total_tiles;
  const uint32_t n_jobs = *M.n_jobs_dev;
  const uint32_t n_split = M.sc.counters[4] < n_jobs ? M.sc.counters[4] : n_jobs;
  const uint64_t split = n_split < n_jobs ? M.prefix[n_split] : total;
  const uint32_t shf = M.cfg.tile_shift;
  // runs of cfg.run tiles amortise claims on big batches; a batch with fewer than two runs per CTA is
  // claimed tile by tile so it spreads over the grid
  const uint32_t kRun = total >= 2ull * gridDim.x * M.cfg.run ? M.cfg.run : 1u;
  const bool map_ok = M.use_map && kRun > 1 && M.sc.counters[13] != 0;
  const uint32_t map_r0 = map_ok ? M.sc.counters[12] : 0;

  if (warp == 0) {
    // ------------------------------------------------ producer
    // Tiles are claimed in runs of kRun consecutive tiles.  The job, its pieces / ring and (decode) the
    // record's fragment table window live in producer-private shared memory: a job is loaded once, and
    // a window of kWin fragment entries is refilled by the whole warp in one round trip, so a tile's
    // descriptor costs no dependent global loads in the common case.
    __shared__ ProdCache pc;
    __shared__ RingDesc ring_s[kMaxRings];  // the index's ring descriptors (decode jobs name their ring)
    if (M.ix.rings)
      for (uint32_t i = lane; i < M.ix.max_rings && i < (uint32_t)kMaxRings; i += 32) ring_s[i] = M.ix.rings[i];
    __syncwarp();
    uint32_t k = 0, claims = 0;
    for (;;) {
      uint64_t t0 = ~0ull, t1 = 0;
      uint32_t run_idx = ~0u;  // index of the claimed run in run_job (when the map applies)
      if (lane == 0) {
        const uint32_t pref = (claims + blockIdx.x) & 1;
        for (int tries = 0; tries < 2 && t0 == ~0ull; ++tries) {
          const uint32_t q = pref ^ tries;
          const uint64_t lo = q ? split : 0, hi = q ? total : split;
          if (lo < hi) {
            // the queue's last cfg.tail tiles per CTA are claimed one at a time (second cursor) so
            // the kernel's tail is one tile, not one run
            const uint64_t tail = (uint64_t)M.cfg.tail * gridDim.x;
            const uint64_t cut = (kRun > 1 && hi - lo > tail) ? lo + (hi - lo - tail) / kRun * kRun : lo;
            uint64_t t = ~0ull;
            uint32_t ri = 0;
            if (cut > lo) { ri = atomicAdd(M.sc.counters + (q ? 2 : 0), 1u); t = lo + (uint64_t)kRun * ri; }
            if (t < cut) {
              t0 = t; t1 = min(cut, t + kRun);
              if (map_ok) run_idx = (q ? map_r0 : 0) + ri;
            } else {
              t = cut + atomicAdd(M.sc.counters + (q ? 6 : 3), 1u);
              if (t < hi) { t0 = t; t1 = t + 1; }
            }
          }
        }
      }
      ++claims;
      t0 = __shfl_sync(0xffffffffu, t0, 0);
      t1 = __shfl_sync(0xffffffffu, t1, 0);
      if (t0 == ~0ull) {
        const uint32_t s = k % kStages;
        StageHdr& H = *reinterpret_cast<StageHdr*>(smem + s * stage_stride);
        mbar_wait(&empty[s], ((k / kStages) & 1) ^ 1);
        if (lane == 0) H.type = JOB_NONE;
        mbar_arrive(&full[s]);
        break;
      }
      uint32_t j;
      run_idx = __shfl_sync(0xffffffffu, run_idx, 0);
      if (run_idx != ~0u) {  // the planner's run -> job map: one load instead of the prefix search
        uint32_t jj = 0;
        if (lane == 0) jj = M.sc.run_job[run_idx];
        j = __shfl_sync(0xffffffffu, jj, 0);
      } else {
        j = find_job(M.prefix, n_jobs, t0, lane);
      }
      uint64_t pj = M.prefix[j], pnext = j + 1 < n_jobs ? M.prefix[j + 1] : ~0ull;
      bool fresh = true;
      for (uint64_t tile = t0; tile < t1; ++tile, ++k) {
        while (tile >= pnext) {  // next job (zero-tile jobs share a prefix value)
          ++j;
          pj = pnext;
          pnext = j + 1 < n_jobs ? M.prefix[j + 1] : ~0ull;
          fresh = true;
        }
        if (fresh) producer_load_job(pc, M, j, lane, ring_s);
        const Job& J = pc.job;
        const uint64_t t = tile - pj;
        const uint64_t A = J.out_start >> shf;
        const uint64_t a = max(J.out_start, (A + t) << shf), b = min(J.out_end, (A + t + 1) << shf);
        uint32_t k0 = 0;
        if (J.type == JOB_DEC) k0 = producer_frag_window(pc, M, J.loff + (a - J.out_start), lane);
        const uint32_t s = k % kStages;
        StageHdr& H = *reinterpret_cast<StageHdr*>(smem + s * stage_stride);
        uint8_t* buf = smem + s * stage_stride + (sizeof(StageHdr) + 127) / 128 * 128;
        mbar_wait(&empty[s], ((k / kStages) & 1) ^ 1);
        // job + pieces into the stage header (shared -> shared)
        if (lane < sizeof(Job) / 4) reinterpret_cast<uint32_t*>(&H.job)[lane] = reinterpret_cast<const uint32_t*>(&J)[lane];
        if (J.type == JOB_ENC)
          for (uint32_t i = lane; i < J.n_pieces * (sizeof(Piece) / 4); i += 32)
            reinterpret_cast<uint32_t*>(H.pieces)[i] = reinterpret_cast<const uint32_t*>(pc.pieces)[i];
        __syncwarp();
        if (lane != 0) mbar_arrive(&full[s]);  // lanes 1-31 are done writing this stage
        if (lane == 0) {
        H.type = J.type;
        H.a = a;
        H.b = b;
        H.fallback = 0;
        H.R = pc.R;
        uint32_t nseg = 0, bytes = 0;
        const uint32_t cap = M.stage_bytes;
        // copies are collected first and issued after expect_tx
        const void* csrc[2 * kMaxSeg];
        uint32_t cdst[2 * kMaxSeg], clen[2 * kMaxSeg], nc = 0;
        auto stage_window = [&](Seg& g, const uint8_t* base, uint64_t mask, bool ring, uint64_t w0, uint64_t w1) {
          // w0..w1: 16-aligned source window (ring cursors or addresses)
          const uint32_t len = (uint32_t)(w1 - w0);
          if (bytes + len > cap) return;
          g.smem_off = bytes;
          g.flags |= 1;
          if (ring) {
            const uint64_t o0 = w0 & mask, cap_r = mask + 1;
            const uint64_t room = cap_r - o0;
            const uint32_t first = room < len ? (uint32_t)room : len;
            csrc[nc] = base + o0; cdst[nc] = bytes; clen[nc] = first; ++nc;
            if (first < len) { csrc[nc] = base; cdst[nc] = bytes + first; clen[nc] = len - first; ++nc; }
          } else {
            csrc[nc] = reinterpret_cast<const void*>(w0); cdst[nc] = bytes; clen[nc] = len; ++nc;
          }
          bytes += len;
        };
        if (J.type == JOB_DEC) {
          H.k0 = k0;
          const uint64_t dst = J.out_start, loff = J.loff;
          uint64_t r = a;
          uint32_t kf = k0;
          bool ok = true;
          while (r < b && kf < pc.nfrags) {
            uint64_t ls, ph;
            uint32_t hd;
            producer_frag(pc, M, kf, ls, ph, hd);
            const uint64_t fl = hd & 0x7fffffffu;
            const uint64_t sb = min(b, dst + (ls + fl - loff));
            if (sb > r) {
              if (nseg == kMaxSeg) { ok = false; break; }
              Seg& g = H.seg[nseg++];
              g.out_a = r;
              g.out_b = sb;
              g.src = ph + (loff + (r - dst) - ls);
              g.flags = (SEG_DATA << 8) | (J.esize << 16);
              const uint64_t c0 = (r + 15) & ~15ull, c1 = sb & ~15ull;
              if (c0 < c1) {  // stage the source window of the interior chunks
                const uint64_t s0 = g.src + (c0 - r);
                const uint64_t w0 = s0 & ~15ull, w1 = (s0 + (c1 - c0) + 15) & ~15ull;
                if (J.esize == 1) {  // bytes: widen the window over the edge bytes (at most 16 B each side)
                  const uint64_t wa = g.src & ~15ull, wb = (g.src + (sb - r) + 15) & ~15ull;
                  stage_window(g, pc.R.base, pc.R.mask, true, wa, wb);
                  if (g.flags & 1) { g.smem_off += (uint32_t)(w0 - wa); g.flags |= 2; }
                } else {
                  stage_window(g, pc.R.base, pc.R.mask, true, w0, w1);
                }
              }
              r = sb;
            }
            ++kf;
          }
          if (!ok) { H.fallback = 1; nseg = 0; nc = 0; bytes = 0; }
        } else if (J.type == JOB_ENC) {
          EncCtx c;
          enc_ctx_init(c, M.sc, J, pc.R, pc.pieces);
          const bool ok = enc_runs(c, a - c.start, b - c.start,
                                   [&](uint32_t kind, uint64_t wa, uint64_t wb, uint64_t src, uint32_t es) {
            if (kind == SEG_LIT && nseg > 0 && (H.seg[nseg - 1].flags >> 8 & 0xff) == SEG_LIT &&
                H.seg[nseg - 1].out_b == c.start + wa) {
              H.seg[nseg - 1].out_b = c.start + wb;  // merge literal runs
              return true;
            }
            if (nseg == kMaxSeg) return false;
            Seg& g = H.seg[nseg++];
            g.out_a = c.start + wa;
            g.out_b = c.start + wb;
            g.src = src;
            g.flags = (kind << 8) | (es << 16);
            if (kind == SEG_DATA) {
              const uint64_t c0 = (g.out_a + 15) & ~15ull, c1 = g.out_b & ~15ull;
              if (c0 < c1) {
                const uint64_t s0 = src + (c0 - g.out_a);
                const uint64_t w0 = s0 & ~15ull, w1 = (s0 + (c1 - c0) + 15) & ~15ull;
                if (es == 1) {  // bytes: widen over the edge bytes (16-byte granules never cross a page)
                  const uint64_t wa = src & ~15ull, wb = (src + (g.out_b - g.out_a) + 15) & ~15ull;
                  stage_window(g, nullptr, 0, false, wa, wb);
                  if (g.flags & 1) { g.smem_off += (uint32_t)(w0 - wa); g.flags |= 2; }
                } else {
                  stage_window(g, nullptr, 0, false, w0, w1);
                }
              }
            }
            return true;
          });
          if (!ok) { H.fallback = 1; nseg = 0; nc = 0; bytes = 0; }
        }
        H.nseg = nseg;
        if (bytes) {
          mbar_arrive_expect_tx(&full[s], bytes);
          for (uint32_t i = 0; i < nc; ++i) bulk_g2s(buf + cdst[i], csrc[i], clen[i], &full[s]);
        } else {
          mbar_arrive(&full[s]);
        }
        }
        fresh = false;
        __syncwarp();
      }
    }
  } else {
    // ------------------------------------------------ consumers
    Team T;
    T.tid = threadIdx.x - 32;
    T.nthr = 32 * kConsumerWarps;
    T.warp = warp - 1;
    T.nwarps = kConsumerWarps;
    for (uint32_t k = 0;; ++k) {
      const uint32_t s = k % kStages;
      const StageHdr& H = *reinterpret_cast<const StageHdr*>(smem + s * stage_stride);
      const uint8_t* buf = smem + s * stage_stride + (sizeof(StageHdr) + 127) / 128 * 128;
      mbar_wait(&full[s], (k / kStages) & 1);
      const uint32_t type = H.type;
      if (type == JOB_NONE) break;
      const Job J = H.job;
      if (type == JOB_DEC) {
        if (H.fallback) {
          DecCtx c;
          dec_ctx_init(c, M.ix, J);
          dec_tile_generic(T, c, H.a, H.b, H.k0);
        } else {
          for (uint32_t g = 0; g < H.nseg; ++g) {
            const Seg S = H.seg[g];
            const uint32_t es = S.flags >> 16 & 0xff;
            const uint64_t c0 = (S.out_a + 15) & ~15ull, c1 = S.out_b & ~15ull;
            if (!(S.flags & 1)) {  // not staged (stage full): direct loads
              DecCtx c;
              dec_ctx_init(c, M.ix, J);
              dec_segment_direct(T, c, S.out_a, S.out_b, S.src);
              continue;
            }
            const uint64_t s0 = S.src + (c0 - S.out_a);
            staged_chunks(T, buf + S.smem_off, (uint32_t)(s0 & 15), (c1 - c0) >> 4, c0, nullptr, es, true);
            // edge bytes (from the stage when the producer widened the window over them)
            const uint64_t ea = min(S.out_b, c0), eb = max(S.out_a, c1);
            const uint32_t ne = (uint32_t)((ea - S.out_a) + (S.out_b - eb));
            if (T.tid < ne) {
              const uint64_t x = T.tid < ea - S.out_a ? S.out_a + T.tid : eb + (T.tid - (ea - S.out_a));
              uint8_t v;
              if (S.flags & 2) {
                v = buf[(int64_t)S.smem_off + (int64_t)(S.src + (x - S.out_a) - (s0 & ~15ull))];
              } else if (es == 1) {
                v = ring_byte(H.R, S.src + (x - S.out_a));
              } else {
                DecCtx c;
                dec_ctx_init(c, M.ix, J);
                v = dec_exact_byte(c, x);
              }
              *reinterpret_cast<uint8_t*>(x) = v;
            }
          }
        }
      } else {
        EncCtx c;
        enc_ctx_init(c, M.sc, J, H.R, H.pieces);
        if (H.fallback) {
          enc_tile_generic(T, c, H.a - c.start, H.b - c.start);
        } else {
          // (composing the literal runs and data edges per 16-byte chunk instead -- enc_gap_chunks -- measured no
          // PCIe-byte gain for host send rings and cost the pipelined step ~5%: the edges stay byte stores here)
          for (uint32_t g = 0; g < H.nseg; ++g) {
            const Seg S = H.seg[g];
            const uint32_t kind = S.flags >> 8 & 0xff, es = S.flags >> 16 & 0xff;
            if (kind == SEG_LIT) {
              enc_bytes(T, c, S.out_a - c.start, S.out_b - c.start);
              continue;
            }
            if (!(S.flags & 1)) {
              enc_segment_direct(T, c, S.out_a - c.start, S.out_b - c.start, S.src, es);
              continue;
            }
            const uint64_t c0 = (S.out_a + 15) & ~15ull, c1 = S.out_b & ~15ull;
            const uint64_t s0 = S.src + (c0 - S.out_a);
            staged_chunks(T, buf + S.smem_off, (uint32_t)(s0 & 15), (c1 - c0) >> 4, c0, &H.R, es, false);
            if (S.flags & 2) {  // edge bytes of plain data, from the widened stage window
              const uint64_t ea = min(S.out_b, c0), eb = max(S.out_a, c1);
              const uint32_t ne = (uint32_t)((ea - S.out_a) + (S.out_b - eb));
              if (T.tid < ne) {
                const uint64_t x = T.tid < ea - S.out_a ? S.out_a + T.tid : eb + (T.tid - (ea - S.out_a));
                H.R.base[x & H.R.mask] = buf[(int64_t)S.smem_off + (int64_t)(S.src + (x - S.out_a) - (s0 & ~15ull))];
              }
            } else {
              enc_bytes(T, c, S.out_a - c.start, min(S.out_b, c0) - c.start);
              enc_bytes(T, c, max(S.out_a, c1) - c.start, S.out_b - c.start);
            }
          }
        }
      }
      mbar_arrive(&empty[s]);  // every consumer thread releases the stage after its last read of it
    }
  }
#ifdef CRK_TIMELINE
  __syncthreads();
#endif
  TL_END(M.cfg, TL_MOVE);
}

// The run -> job map of the next mover launch (grid CTAs, runs of `run` tiles, cfg.tail tail tiles per CTA):
// the run boundaries are the mover's own (queue 0 = decode jobs from tile 0, queue 1 = encode jobs from the
// split, runs up to the queue's single-tile tail region); each thread maps one run by binary search over
// the tile prefix.  counters[12] = queue-0 run count, counters[13] = 1 when the map applies.
__global__ void run_map_kernel(Scratch sc, ConfigDev cfg, uint32_t grid, uint32_t run, const uint64_t* prefix,
                               const uint32_t* n_jobs_dev, const uint64_t* total_tiles) {
  pdl_entry();
  const uint64_t total = *total_tiles;
  const uint32_t n_jobs = *n_jobs_dev;
  const uint32_t n_split = sc.counters[4] < n_jobs ? sc.counters[4] : n_jobs;
  const uint64_t split = n_split < n_jobs ? prefix[n_split] : total;
  const uint32_t kRun = total >= 2ull * grid * run ? run : 1u;
  const uint64_t tail = (uint64_t)cfg.tail * grid;
  auto runs_of = [&](uint64_t lo, uint64_t hi) -> uint64_t {
    const uint64_t cut = (kRun > 1 && hi - lo > tail) ? lo + (hi - lo - tail) / kRun * kRun : lo;
    return (cut - lo) / kRun;
  };
  const uint64_t r0 = split > 0 ? runs_of(0, split) : 0, r1 = total > split ? runs_of(split, total) : 0;
  const bool ok = kRun > 1 && r0 + r1 <= sc.max_jobs;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    sc.counters[12] = (uint32_t)r0;
    sc.counters[13] = ok ? 1u : 0u;
  }
  if (!ok) return;
  for (uint64_t r = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; r < r0 + r1; r += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t t = r < r0 ? r * kRun : split + (r - r0) * kRun;
    uint32_t lo = 0, hi = n_jobs;  // last j with prefix[j] <= t (zero-tile jobs share a prefix value)
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (prefix[mid] <= t) lo = mid; else hi = mid;
    }
    sc.run_job[r] = lo;
  }
}

// tiles per job: output range cut at tile_bytes-aligned boundaries
__global__ void plan_count_kernel(Scratch sc, ConfigDev cfg, uint64_t* tiles, const uint32_t* n_jobs_dev) {
  pdl_entry();
  const uint32_t n = *n_jobs_dev;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    sc.counters[0] = 0;  // decode-queue run cursor
    sc.counters[2] = 0;  // encode-queue run cursor
    sc.counters[3] = 0;  // decode-queue tail (single-tile) cursor
    sc.counters[6] = 0;  // encode-queue tail cursor
  }
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n; j += gridDim.x * blockDim.x) {
    const Job jb = sc.jobs[j];
    uint64_t c = 0;
    if (jb.type != JOB_NONE && jb.out_end > jb.out_start)
      c = ((jb.out_end - 1) >> cfg.tile_shift) - (jb.out_start >> cfg.tile_shift) + 1;
    tiles[j] = c;
  }
}

// Small requests (<= kSmallJobs jobs): tile counts, their exclusive prefix (K2 in one block) and the
// cursor reset in a single launch.
constexpr uint32_t kSmallJobs = 2048;
__global__ void __launch_bounds__(256) plan_small_kernel(Scratch sc, ConfigDev cfg, uint64_t* tiles, uint64_t* total,
                                                         const uint32_t* n_jobs_dev) {
  pdl_entry();
  __shared__ uint64_t warp_sum[8];
  const uint32_t n = *n_jobs_dev;
  if (threadIdx.x == 0) {
    sc.counters[0] = 0;
    sc.counters[2] = 0;
    sc.counters[3] = 0;
    sc.counters[6] = 0;
  }
  constexpr uint32_t IPT = kSmallJobs / 256;
  uint64_t v[IPT], acc = 0;
#pragma unroll
  for (uint32_t i = 0; i < IPT; ++i) {
    const uint32_t j = threadIdx.x * IPT + i;
    uint64_t c = 0;
    if (j < n) {
      const Job jb = sc.jobs[j];
      if (jb.type != JOB_NONE && jb.out_end > jb.out_start)
        c = ((jb.out_end - 1) >> cfg.tile_shift) - (jb.out_start >> cfg.tile_shift) + 1;
    }
    v[i] = c;
    acc += c;
  }
  const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint64_t x = acc;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint64_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= (uint32_t)o) x += y;
  }
  if (lane == 31) warp_sum[w] = x;
  __syncthreads();
  uint64_t base = 0;
  for (uint32_t i = 0; i < w; ++i) base += warp_sum[i];
  uint64_t run = base + x - acc;
#pragma unroll
  for (uint32_t i = 0; i < IPT; ++i) {
    const uint32_t j = threadIdx.x * IPT + i;
    if (j < n) tiles[j] = run;
    run += v[i];
  }
  if (threadIdx.x == 255) *total = run;
}

}  // namespace

uint32_t mover_smem_bytes(uint32_t tile_bytes, uint32_t kStages) {
  const uint32_t stage_bytes = tile_bytes + 32 * kMaxSeg + 32;
  return kStages * ((uint32_t)(sizeof(StageHdr) + 127) / 128 * 128 + stage_bytes);
}

cudaError_t launch_plan_and_move(const IndexDev* ix, const ConfigDev& cfg, Scratch& sc, uint32_t max_jobs_bound,
                                 uint64_t out_bytes_bound, int sms, int move_ctas, cudaStream_t s, bool planned) {
  uint64_t* tiles = sc.scan_tmp;  // [max_jobs + 1]
  uint64_t* total = sc.scan_tmp + sc.max_jobs + 1;
  const uint32_t* n_jobs_dev = sc.counters + 1;
  cudaError_t e;
  if (planned) {
  } else if (max_jobs_bound <= kSmallJobs) {
    CRK_LAUNCH(pdl_of(cfg), plan_small_kernel, 1, 256, 0, s, sc, cfg, tiles, total, n_jobs_dev);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
  } else {
    const uint32_t cnt_blocks = (max_jobs_bound + 255) / 256;
    CRK_LAUNCH(pdl_of(cfg), plan_count_kernel, min(cnt_blocks, (uint32_t)sms * 8), 256, 0, s, sc, cfg, tiles, n_jobs_dev);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    e = launch_exclusive_scan_u64(tiles, max_jobs_bound, n_jobs_dev, total, sc, s);
    if (e != cudaSuccess) return e;
  }
  // a known bound on the output bytes caps the grid at the tiles that can exist
  uint32_t run = cfg.run;
  if (out_bytes_bound) {
    const uint64_t tiles_max = 2ull * max_jobs_bound + (out_bytes_bound >> cfg.tile_shift) + 1;
    if (tiles_max < (uint64_t)move_ctas * run) {
      run = 1;  // few tiles: one per claim, spread over the CTAs
      if (tiles_max < (uint64_t)move_ctas) move_ctas = (int)tiles_max;
    }
  }
  bool use_map = false;
  if (!planned && run > 1) {  // the run -> job map for this launch's run boundaries
    CRK_LAUNCH(pdl_of(cfg), run_map_kernel, (uint32_t)sms * 2, 256, 0, s, sc, cfg, (uint32_t)move_ctas, run, tiles, n_jobs_dev, total);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    use_map = true;
  }
  return launch_mover(ix, cfg, sc, run, move_ctas, s, use_map);
}

// The mover over already-planned jobs: tile prefix in scan_tmp[0..n_jobs), total tiles at
// scan_tmp[max_jobs + 1], job count in counters[1], queue split in counters[4], cursors reset.
cudaError_t launch_mover(const IndexDev* ix, const ConfigDev& cfg, Scratch& sc, uint32_t run, int move_ctas,
                         cudaStream_t s, bool use_map) {
  cudaError_t e;
  MoveParams M;
  if (ix) M.ix = *ix; else memset(&M.ix, 0, sizeof(M.ix));
  M.sc = sc;
  M.cfg = cfg;
  M.cfg.run = run;
  M.prefix = sc.scan_tmp;
  M.n_jobs_dev = sc.counters + 1;
  M.total_tiles = sc.scan_tmp + sc.max_jobs + 1;
  M.stage_bytes = (1u << cfg.tile_shift) + 32 * kMaxSeg + 32;
  M.seq = ++sc.mover_seq;
  M.use_map = use_map ? 1u : 0u;
  M.opp_from = (uint32_t)move_ctas > 2 * cfg.reserve ? (uint32_t)move_ctas - cfg.reserve : (uint32_t)move_ctas;
  // Reserved CTAs compare against the launch stamp of the same launch (sequence M.seq).  A captured graph
  // replays one baked M.seq, so a replay could read the previous replay's stamp: no reserve under capture.
  cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
  if (cudaStreamIsCapturing(s, &cap) == cudaSuccess && cap != cudaStreamCaptureStatusNone)
    M.opp_from = (uint32_t)move_ctas;
  const uint32_t smem = mover_smem_bytes(1u << cfg.tile_shift, cfg.stages);
  if ((e = ensure_mover_smem(smem)) != cudaSuccess) return e;
  prof_mark(PROF_MOVE, true, s);
  {
    // Not early-scheduled when it keeps reserved CTAs (a pipelined server loop): CTAs resident early would sit
    // on SM slots the next batch's front end needs, and would all pass the launch-time gate at once.
    const cudaError_t le = launch_k_opt(cfg.reserve == 0, mover_kernel, move_ctas, kMoverThreads, smem, s, M);
    if (le != cudaSuccess) return le;
  }
  prof_mark(PROF_MOVE, false, s);
  return cudaGetLastError();
}

// The mover's dynamic shared memory opt-in is a per-device attribute of the kernel.  It is kept per device
// and only ever raised (under a lock), so a context created later with smaller tiles never lowers the
// limit another context's launches rely on, and each device gets its own opt-in.
cudaError_t ensure_mover_smem(uint32_t smem) {
  static std::mutex mu;
  static uint32_t set[kMaxDevices] = {};
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= kMaxDevices) return cudaErrorInvalidDevice;
  std::lock_guard<std::mutex> lk(mu);
  if (smem <= set[dev]) return cudaSuccess;
  e = cudaFuncSetAttribute(mover_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess) set[dev] = smem;
  return e;
}

// CTAs per SM the mover can keep resident for a tile size (raises the dynamic shared memory limit).
int mover_occupancy(uint32_t tile_bytes, uint32_t stages) {
  const uint32_t smem = mover_smem_bytes(tile_bytes, stages);
  if (ensure_mover_smem(smem) != cudaSuccess) return 0;
  int n = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, mover_kernel, kMoverThreads, smem);
  return n;
}

}  // namespace crk
