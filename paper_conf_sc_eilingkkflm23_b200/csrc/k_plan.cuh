// Serve planning helpers (oracle or_serve decisions, reply jobs, block sums) shared by the planning
// kernels (k_plan.cu) and the persistent server (k_server.cu).
#pragma once
#include "crk_device.cuh"

namespace crk {

namespace {

constexpr uint32_t kNotFound = 0xffffffffu;

__device__ __forceinline__ uint32_t elem_size_k(uint32_t kind) {
  switch (kind) {
    case CRK_K_OPAQUE_VAR: case CRK_K_OPAQUE_FIX: return 1;
    case CRK_K_I32_VAR: case CRK_K_U32_VAR: case CRK_K_F32_VAR:
    case CRK_K_I32_FIX: case CRK_K_U32_FIX: case CRK_K_F32_FIX: return 4;
    case CRK_K_I64_VAR: case CRK_K_U64_VAR: case CRK_K_F64_VAR:
    case CRK_K_I64_FIX: case CRK_K_U64_FIX: case CRK_K_F64_FIX: return 8;
    default: return 0;
  }
}

// xid -> dense id of the earliest record carrying it (reading R11)
__device__ __forceinline__ uint32_t xid_lookup(const IndexDev& ix, uint32_t xid) {
  uint32_t h = (xid * 0x9E3779B1u) & ix.hash_mask;
  for (;;) {
    const unsigned long long k = ix.xid_hash[h];
    if (k == ~0ull) return kNotFound;
    if ((uint32_t)(k >> 32) == xid) return (uint32_t)k;
    h = (h + 1) & ix.hash_mask;
  }
}

__device__ __forceinline__ uint64_t wire_of(uint64_t Ll, uint32_t F) {
  const uint64_t nfr = Ll == 0 ? 1 : (Ll + F - 1) / F;  // reading R3: >= 1 fragment, no empty trailer
  return Ll + 4 * nfr;
}

// A decode job carries its record's fragment-table coordinates (first fragment, count, ring, first
// fragment length), so the mover's producer resolves a fresh job with one load instead of a chain of
// record-table loads.
// Its coordinates are the parser's per-record copies (p_frag0 / p_nfrags / p_flen0 / p_ring): one round trip.
struct RecCoord {
  uint32_t frag0, nfrags, flen0, ring;
};
__device__ __forceinline__ RecCoord rec_coord(const IndexDev& ix, uint32_t rec) {
  return RecCoord{ix.p_frag0[rec], ix.p_nfrags[rec], ix.p_flen0[rec], ix.p_ring[rec]};
}
__device__ __forceinline__ Job dec_job(const RecCoord& rc, uint64_t dst, uint64_t nbytes, uint64_t loff, uint32_t rec,
                                       uint32_t es) {
  Job j{};
  j.type = nbytes ? JOB_DEC : JOB_NONE;
  j.esize = es;
  j.rec = rec;
  j.out_start = dst;
  j.out_end = dst + nbytes;
  j.loff = loff;
  if (nbytes) {
    j.piece0 = rc.frag0;
    j.n_pieces = rc.nfrags;
    j.out_ring = rc.ring;
    j.F = rc.flen0;
  }
  return j;
}
__device__ __forceinline__ Job dec_job(const IndexDev& ix, uint64_t dst, uint64_t nbytes, uint64_t loff, uint32_t rec,
                                       uint32_t es) {
  return dec_job(rec_coord(ix, rec), dst, nbytes, loff, rec, es);
}

// ---- serve: statuses, HtoD decode jobs and reply sizes (pass 1) --------------------------------
__device__ __forceinline__ void reply_words(Piece& p, uint32_t xid, int32_t err, bool with_len, uint64_t n) {
  p = Piece{};
  p.type = PIECE_WORDS;
  p.loff = 0;
  p.words[0] = xid;  // RFC 5531 §9: xid, REPLY, MSG_ACCEPTED, verf AUTH_NONE (0, len 0), SUCCESS
  p.words[1] = 1;
  p.words[2] = 0;
  p.words[3] = 0;
  p.words[4] = 0;
  p.words[5] = 0;
  p.words[6] = (uint32_t)err;  // mem_result discriminant (reading R10)
  if (with_len) p.words[7] = (uint32_t)n;
  p.nbytes = with_len ? 32 : 28;
}

// ---- striped memcpys (reading R22): the parent table of a serve step ------------------------------------
// An OK stripe of `parent` adds its bytes; the first OK stripe claims (ptr, total), a disagreeing one marks the
// parent inconsistent; a stripe at offset 0 offers itself as the lead (smallest dense id).
__device__ __forceinline__ void stripe_add(const IndexDev& ix, uint32_t parent, uint64_t ptr, uint64_t total,
                                           uint64_t m, bool at0, uint32_t d) {
  uint32_t h = (parent * 0x9E3779B1u) & ix.hash_mask;
  for (;;) {
    StripeEnt& e = ix.stripe[h];
    const unsigned long long k = atomicCAS(&e.key, ~0ull, (unsigned long long)parent);
    if (k == ~0ull) ix.stripe_list[atomicAdd(ix.stripe_n, 1u)] = h;  // a new parent: remember its slot
    if (k == ~0ull || k == parent) {
      const unsigned long long p0 = atomicCAS(&e.ptr, ~0ull, (unsigned long long)ptr);
      const unsigned long long t0 = atomicCAS(&e.total, ~0ull, (unsigned long long)total);
      if ((p0 != ~0ull && p0 != ptr) || (t0 != ~0ull && t0 != total)) atomicAnd(&e.good, 0u);
      atomicAdd(&e.landed_c, (unsigned long long)(0ull - m));  // ~landed - m = ~(landed + m)
      if (at0) atomicMin(&e.lead, d);
      return;
    }
    h = (h + 1) & ix.hash_mask;
  }
}

// True when stripe record d (OK, at offset 0) leads a complete parent: consistent, every byte landed.
__device__ __forceinline__ bool stripe_leads(const IndexDev& ix, uint32_t parent, uint32_t d) {
  uint32_t h = (parent * 0x9E3779B1u) & ix.hash_mask;
  for (;;) {
    const StripeEnt* e = ix.stripe + h;
    const unsigned long long k = __ldcg(&e->key);
    if (k == ~0ull) return false;
    if (k == parent)
      return __ldcg(&e->lead) == d && __ldcg(&e->good) != 0 && ~__ldcg(&e->landed_c) == __ldcg(&e->total);
    h = (h + 1) & ix.hash_mask;
  }
}

// Resets the parent slots a step used (entries [i0, n) of the list, stride st) to the empty state.
__device__ __forceinline__ void stripe_clear(const IndexDev& ix, uint32_t n, uint32_t i0, uint32_t st) {
  for (uint32_t i = i0; i < n; i += st) {
    StripeEnt& e = ix.stripe[ix.stripe_list[i]];
    e.key = e.ptr = e.total = e.landed_c = ~0ull;
    e.lead = e.good = ~0u;
  }
}

// Serve decisions for dense record d (oracle or_serve): final status, reply discriminant (-1: no reply),
// reply logical length, and the HtoD decode job.  A striped memcpy's stripe (reading R22) decides like an
// HtoD copy to ptr + offset with no reply; whether the offset-0 stripe carries its parent's reply is known
// only once every stripe of the step has decided (stripe_leads, after a block / grid barrier).
// `sole`: d is the step's only record, so it owns its xid without a lookup.
__device__ __forceinline__ void serve_decide(const IndexDev& ix, const ConfigDev& cfg, uint32_t d, uint64_t region_base,
                                             uint64_t region_bytes, int& st, int32_t& err, uint64_t& Ll, Job& job,
                                             bool sole = false) {
  // every field the decision can need is loaded at once (one memory round trip), then the xid lookup
  const uint64_t b = (uint64_t)d * kMaxItems;
  st = ix.p_status[d];
  const uint32_t proc = ix.p_proc[d], xid = ix.p_xid[d];
  const uint64_t v0 = ix.p_value[b], v1 = ix.p_value[b + 1], v2 = ix.p_value[b + 2];
  const uint64_t c1 = ix.p_count[b + 1], o1 = ix.p_off[b + 1];
  const RecCoord rc = rec_coord(ix, d);
  err = -1;
  Ll = 0;
  job = Job{};
  if (st == CRK_OK && !sole && xid_lookup(ix, xid) != d) st = CRK_E_XID;
  if (st == CRK_OK && proc == cfg.proc_h2d) {
    const uint64_t ptr = v0, nb = c1, size = v2;
    const uint64_t m = (cfg.strict || nb <= size) ? nb : size;
    if (cfg.strict && nb != size) { st = CRK_E_SIZE; err = 1; }
    else if (ptr < region_base || m > region_bytes || ptr - region_base > region_bytes - m) { st = CRK_E_PTR; err = 1; }
    else { err = 0; job = dec_job(rc, ptr, m, o1, d, 1); }
    Ll = 28;
  } else if (st == CRK_OK && cfg.proc_stripe && proc == cfg.proc_stripe) {
    const uint64_t v3 = ix.p_value[b + 3], off = ix.p_value[b + 4], tot = ix.p_value[b + 5];
    const uint64_t nb = c1, size = v2;
    const uint64_t m = (cfg.strict || nb <= size) ? nb : size;
    if (cfg.strict && nb != size) st = CRK_E_SIZE;
    else if (tot >= (1ull << 63) || off > tot || m > tot - off) st = CRK_E_SIZE;
    else if (v0 > ~0ull - off) st = CRK_E_PTR;
    else {
      const uint64_t ptr = v0 + off;
      if (ptr < region_base || m > region_bytes || ptr - region_base > region_bytes - m) st = CRK_E_PTR;
      else {
        job = dec_job(rc, ptr, m, o1, d, 1);
        stripe_add(ix, (uint32_t)v3, v0, tot, m, off == 0, d);
        Ll = 28;  // the parent's reply, if this stripe turns out to lead a complete memcpy
      }
    }
  } else if (st == CRK_OK && proc == cfg.proc_d2h) {
    const uint64_t ptr = v0, size = v1;
    if (size > 0xffffffffull || ptr < region_base || size > region_bytes || ptr - region_base > region_bytes - size) {
      st = CRK_E_PTR; err = 1; Ll = 28;
    } else {
      err = 0; Ll = 32 + size + pad4(size);
    }
  }
}

// The reply of record d as an encode job (pieces at 2d, 2d+1) written at send-ring cursor `off`.
__device__ __forceinline__ Job serve_reply_job(const IndexDev& ix, const ConfigDev& cfg, const Scratch& sc, uint32_t d,
                                               uint32_t ring, int32_t err, uint64_t off, uint64_t w) {
  Job job{};
  if (err < 0) return job;
  const uint64_t b = (uint64_t)d * kMaxItems;
  const uint32_t proc = ix.p_proc[d];
  const bool d2h = proc == cfg.proc_d2h && err == 0;
  const uint64_t n = d2h ? ix.p_value[b + 1] : 0;
  // a striped memcpy's reply carries the parent memcpy's xid (reading R22)
  const uint32_t xid = (cfg.proc_stripe && proc == cfg.proc_stripe) ? (uint32_t)ix.p_value[b + 3] : ix.p_xid[d];
  Piece* P = sc.pieces + 2ull * d;
  reply_words(P[0], xid, err, d2h, n);
  uint32_t np = 1;
  uint64_t Ll = P[0].nbytes;
  if (d2h) {
    Piece q{};
    q.type = PIECE_DATA;
    q.loff = 32;
    q.nbytes = n;
    q.src = ix.p_value[b];
    q.esize = 1;
    P[1] = q;
    np = 2;
    Ll = 32 + n + pad4(n);
  }
  job.type = JOB_ENC;
  job.out_start = off;
  job.out_end = off + w;
  job.loff = Ll;
  job.piece0 = 2 * d;
  job.n_pieces = np;
  job.F = cfg.F;
  job.out_ring = ring;
  return job;
}

// The mover plan of a single job, written by the thread that built it (single-request calls skip the
// separate planning launch): tile prefix [0] = 0, total tiles, queue cursors reset.
__device__ __forceinline__ void plan_single_job(const Scratch& sc, const ConfigDev& cfg, const Job& j) {
  const uint64_t t = (j.type == JOB_NONE || j.out_end <= j.out_start)
                         ? 0 : ((j.out_end - 1) >> cfg.tile_shift) - (j.out_start >> cfg.tile_shift) + 1;
  sc.scan_tmp[0] = 0;
  sc.scan_tmp[sc.max_jobs + 1] = t;
  sc.counters[0] = 0;
  sc.counters[2] = 0;
  sc.counters[3] = 0;
  sc.counters[6] = 0;
}

struct SendRingsParam {
  uint32_t n_rings;
  RingDesc r[kMaxRings];
  uint64_t off[kMaxRings];
  const uint64_t* doorbell;  // if set, send offsets are doorbell[2 * n_rings + r]
};

// Block-wide exclusive sums of NV values per thread at once (blockDim.x threads, a multiple of 32, <= 1024):
// warp shuffle scans, then warp 0 scans the warp totals (no per-thread loop over the 32 warp sums, which cost
// ~0.5 us of dependent shared-memory loads per scan in a 1024-thread block).  warp_sums: NV x 32 entries.
// Returns the block totals through tot[].
template <int NV>
__device__ __forceinline__ void block_excl_sums(uint64_t (&v)[NV], uint64_t* warp_sums, uint64_t (&tot)[NV]) {
  const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  uint64_t x[NV];
#pragma unroll
  for (int k = 0; k < NV; ++k) x[k] = v[k];
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
#pragma unroll
    for (int k = 0; k < NV; ++k) {
      const uint64_t y = __shfl_up_sync(0xffffffffu, x[k], o);
      if (lane >= (uint32_t)o) x[k] += y;
    }
  }
  cta_barrier();
  if (lane == 31)
#pragma unroll
    for (int k = 0; k < NV; ++k) warp_sums[32 * k + w] = x[k];
  cta_barrier();
  if (w == 0) {  // inclusive prefix of the warp totals, in place
#pragma unroll
    for (int k = 0; k < NV; ++k) {
      uint64_t y = lane < nw ? warp_sums[32 * k + lane] : 0;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint64_t z = __shfl_up_sync(0xffffffffu, y, o);
        if (lane >= (uint32_t)o) y += z;
      }
      if (lane < nw) warp_sums[32 * k + lane] = y;
    }
  }
  cta_barrier();
#pragma unroll
  for (int k = 0; k < NV; ++k) {
    tot[k] = warp_sums[32 * k + nw - 1];
    v[k] = (w ? warp_sums[32 * k + w - 1] : 0) + x[k] - v[k];
  }
}
__device__ __forceinline__ uint64_t block_excl_sum(uint64_t v, uint64_t* warp_sums, uint64_t* tot) {
  uint64_t a[1] = {v}, t[1];
  block_excl_sums<1>(a, warp_sums, t);
  *tot = t[0];
  return a[0];
}

// The same exclusive sums over one warp (no block barrier): tot[] = the warp totals.
template <int NV>
__device__ __forceinline__ void warp_excl_sums(uint64_t (&v)[NV], uint64_t (&tot)[NV]) {
  const uint32_t lane = threadIdx.x & 31;
  uint64_t x[NV];
#pragma unroll
  for (int k = 0; k < NV; ++k) x[k] = v[k];
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
#pragma unroll
    for (int k = 0; k < NV; ++k) {
      const uint64_t y = __shfl_up_sync(0xffffffffu, x[k], o);
      if (lane >= (uint32_t)o) x[k] += y;
    }
  }
#pragma unroll
  for (int k = 0; k < NV; ++k) {
    tot[k] = __shfl_sync(0xffffffffu, x[k], 31);
    v[k] = x[k] - v[k];
  }
}

#ifdef CRK_PLAN_TRACE
// Diagnostic build only: %globaltimer at the sub-phases of plan_small_block (thread 0), per translation unit.
__device__ unsigned long long g_plan_trace[16];
#define PLAN_MARK(i) do { if (threadIdx.x == 0) { unsigned long long t_; \
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_)); g_plan_trace[i] = t_; } } while (0)
#else
#define PLAN_MARK(i) do { } while (0)
#endif

// Small batches (<= kSmallServe records): statuses, reply offsets, decode and encode jobs, their tile
// prefix and the mover cursors, by one block of kSmallServe threads (thread d owns record d).
// warp_sums (32) and ring_first_pre (kMaxRings) are the block's shared scratch.  Used by the
// single-block planning kernel, the fused front end and the persistent server; the latter two pass the
// dense record prefix they already hold in shared memory (prefix_s, n_rings + 1 entries), which saves the
// dependent loads of the record total and of each record's ring bounds.  kOneWarp: a step of at most 32
// records is planned by warp 0 alone, its sums by shuffles, with no block barrier.
// Optional shared-memory copies of the plan for a caller that moves the step itself (the persistent server):
// the jobs (when 2 * total <= cap), the tile total and each ring's reply bytes, so its move phase needs no
// load of what the plan just wrote.  reply_bytes must hold 0 for every ring beforehand.
struct PlanOut {
  Job* jobs;
  uint32_t cap;
  uint64_t* tiles;
  uint64_t* reply_bytes;
};

template <bool kOneWarp>
__device__ void plan_small_impl(const IndexDev& ix, const ConfigDev& cfg, const Scratch& sc, const SendRingsParam& S,
                                uint64_t region_base, uint64_t region_bytes, uint64_t* warp_sums,
                                uint64_t* ring_first_pre, const uint32_t* prefix_s, uint32_t total,
                                const PlanOut* out) {
  PLAN_MARK(0);
  const uint32_t d = threadIdx.x, nthreads = kOneWarp ? 32u : blockDim.x;
  for (uint32_t r = threadIdx.x; r < S.n_rings; r += nthreads) sc.out_rings[r] = S.r[r];
  int st = CRK_OK;
  int32_t err = -1;
  uint64_t Ll = 0, w = 0;
  Job dec{};
  uint32_t ring = 0, first = 0, end = 0;
  if (d < total) {
    ring = ix.p_ring[d];
    serve_decide(ix, cfg, d, region_base, region_bytes, st, err, Ll, dec, total == 1);
    first = prefix_s ? prefix_s[ring] : ix.rec_prefix[ring];
    end = prefix_s ? prefix_s[ring + 1] : ix.rec_prefix[ring + 1];
  }
  PLAN_MARK(1);
  // every stripe of the step has decided: the leads of complete memcpys reply (the block-wide OR of "an OK
  // stripe here" skips the parent table altogether in steps without stripes)
  const bool my_stripe = cfg.proc_stripe && d < total && st == CRK_OK && Ll == 28 && err < 0;  // only OK stripes
  if (kOneWarp) __syncwarp();  // orders the warp's parent-table atomics before the leads read the table
  const bool any_stripe =
      cfg.proc_stripe && (kOneWarp ? __any_sync(0xffffffffu, my_stripe) : cta_barrier_or(my_stripe));
  if (my_stripe && stripe_leads(ix, (uint32_t)ix.p_value[(uint64_t)d * kMaxItems + 3], d)) err = 0;
  if (d < total) w = err >= 0 ? wire_of(Ll, cfg.F) : 0;
  PLAN_MARK(2);
  uint64_t tot, pre;
  if (kOneWarp) {  // reply sizes -> offsets
    uint64_t a[1] = {w}, t[1];
    warp_excl_sums<1>(a, t);
    pre = a[0];
    tot = t[0];
  } else {
    pre = block_excl_sum(w, warp_sums, &tot);
  }
  (void)tot;
  if (d < total && d == first) ring_first_pre[ring] = pre;
  if (kOneWarp) __syncwarp(); else cta_barrier();
  PLAN_MARK(3);
  Job enc{};
  if (d < total) {
    const uint64_t off = (S.doorbell ? S.doorbell[2 * S.n_rings + ring] : S.off[ring]) + (pre - ring_first_pre[ring]);
    ix.s_status[d] = st;
    ix.s_reply_err[d] = err;
    ix.s_reply_wire[d] = w;
    ix.s_reply_off[d] = err >= 0 ? off : 0;  // (the oracle's convention: 0 when the record has no reply)
    enc = serve_reply_job(ix, cfg, sc, d, ring, err, off, w);
    sc.jobs[d] = dec;
    sc.jobs[total + d] = enc;
    if (d + 1 == end) ix.res[ring].reply_bytes = pre + w - ring_first_pre[ring];
    if (out) {
      if (2 * total <= out->cap) {
        out->jobs[d] = dec;
        out->jobs[total + d] = enc;
      }
      if (d + 1 == end) out->reply_bytes[ring] = pre + w - ring_first_pre[ring];
    }
  }
  // mover plan: tiles per job (decode jobs [0, total), encode jobs [total, 2 total)) and their prefix
  auto tiles_of = [&](const Job& j) -> uint64_t {
    if (j.type == JOB_NONE || j.out_end <= j.out_start) return 0;
    return ((j.out_end - 1) >> cfg.tile_shift) - (j.out_start >> cfg.tile_shift) + 1;
  };
  PLAN_MARK(4);
  __shared__ uint64_t ws2[64];
  uint64_t tv[2] = {d < total ? tiles_of(dec) : 0, d < total ? tiles_of(enc) : 0}, tt[2];
  if (kOneWarp) warp_excl_sums<2>(tv, tt);
  else block_excl_sums<2>(tv, ws2, tt);  // decode and encode tile counts in one pass
  const uint64_t pd = tv[0], pe = tv[1], tot_d = tt[0], tot_e = tt[1];
  if (d < total) {
    sc.scan_tmp[d] = pd;
    sc.scan_tmp[total + d] = tot_d + pe;
  }
  PLAN_MARK(5);
  if (any_stripe) {  // leave the parent table empty for the next step (every lead has read it)
    const uint32_t n = __ldcg(ix.stripe_n);
    stripe_clear(ix, n, threadIdx.x, nthreads);
    if (kOneWarp) __syncwarp(); else cta_barrier();
    if (d == 0 && n) *ix.stripe_n = 0;
  }
  if (d == 0) {
    if (out) *out->tiles = tot_d + tot_e;
    sc.scan_tmp[sc.max_jobs + 1] = tot_d + tot_e;
    sc.counters[0] = 0;
    sc.counters[2] = 0;
    sc.counters[3] = 0;
    sc.counters[6] = 0;
    sc.counters[1] = 2 * total;
    sc.counters[4] = total;
  }
  PLAN_MARK(6);
}

__device__ void plan_small_block(const IndexDev& ix, const ConfigDev& cfg, const Scratch& sc, const SendRingsParam& S,
                                 uint64_t region_base, uint64_t region_bytes, uint64_t* warp_sums,
                                 uint64_t* ring_first_pre, const uint32_t* prefix_s = nullptr,
                                 const PlanOut* out = nullptr) {
  const uint32_t total = prefix_s ? prefix_s[S.n_rings] : *ix.total;
  if (total <= 32) {
    if (threadIdx.x < 32)
      plan_small_impl<true>(ix, cfg, sc, S, region_base, region_bytes, warp_sums, ring_first_pre, prefix_s, total,
                            out);
  } else {
    plan_small_impl<false>(ix, cfg, sc, S, region_base, region_bytes, warp_sums, ring_first_pre, prefix_s, total,
                           out);
  }
}

}  // namespace
}  // namespace crk
