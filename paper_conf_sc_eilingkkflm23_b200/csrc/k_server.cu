// Persistent server (include/crk.h crk_server_*): one resident CTA polls a
// doorbell and runs each published step with the same device functions as the launched pipeline --
// scan_ring_cta (K1), parse_record (K3), plan_small_block (serve planning), the generic movers (K4-K7) --
// so a small call costs a few dependent memory round trips instead of five kernel launches.
//
// Rings change under a running kernel, so this translation unit reads them with coherent loads
// (CRK_COHERENT_LOADS: ld.global.cg instead of the read-only path).  Each step starts with a system-scope
// acquire of the doorbell (the host's ring writes, and device writes of other streams released before it,
// are visible to every thread after the following barrier).  Phases hand data to each other only inside
// this one CTA, so a block barrier orders them (CUDA memory model: __syncthreads makes the block's prior
// global writes and atomics visible to the block); no device-wide fence per phase (≈1 µs each).
#define CRK_COHERENT_LOADS 1
#include "k_move.cuh"
#include "k_parse.cuh"
#include "k_plan.cuh"
#include "k_scan.cuh"

namespace crk {

namespace {

constexpr uint32_t kServerThreads = kSmallServe;  // plan_small_block: thread d owns record d
constexpr uint32_t kServerWarps = kServerThreads / 32;
static_assert(kMaxRings <= kServerThreads, "thread r < n_rings holds ring r's result");

struct ServerParams {
  IndexDev ix;
  ConfigDev cfg;
  Scratch sc;
  const SchemaTable* schemas;
  crk_server_bell* bell;
  uint32_t n_rings;
  RingDesc rings[kMaxRings];   // base / mask; cursors come from the bell
  RingDesc send[kMaxRings];
  uint64_t region_base, region_bytes;
  uint64_t dev_rings;          // bit r: receive ring r is device memory (its small records are prefetched to L2)
};

__device__ __forceinline__ uint64_t ld_acquire_sys(const volatile uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(volatile uint64_t* p, uint64_t v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// Phase boundary: the block's global writes and atomics of the previous phase are visible to the block.
__device__ __forceinline__ void phase_sync() {
  cta_barrier();
#ifdef CRK_SERVER_PHASE_FENCE  // diagnostic: a device-wide fence per phase as well
  if (threadIdx.x == 0) __threadfence();
  cta_barrier();
#endif
}

// Moves output tile t (2^sh-aligned in output space, like the mover's tiles) of job J with team T
// (generic paths of k_move.cuh).
// tiles dealt to the warps round-robin: 2 KiB (one chunk-loop pass per warp) when the step moves at most
// ~4 mover tiles' worth of bytes, else 8 KiB
#ifndef CRK_SERVER_POLLERS
#define CRK_SERVER_POLLERS 1
#endif
constexpr uint32_t kPollers = CRK_SERVER_POLLERS;  // warps whose lane 0 polls the doorbell (A/B on one B200: 4 staggered
                                                   // pollers 18.1 us round trip per 4 KiB call vs 16.0 for one)
constexpr uint64_t kPrefetchMax = 64 * 1024;  // records up to this size have their payload prefetched to L2
constexpr uint32_t kJobCache = 32;   // jobs staged in shared memory at the start of the move phase
__device__ __forceinline__ uint64_t job_tiles(const Job& J, uint32_t sh) {
  if (J.type == JOB_NONE || J.out_end <= J.out_start) return 0;
  return ((J.out_end - 1) >> sh) - (J.out_start >> sh) + 1;
}
__device__ __forceinline__ void move_tile(const Team& T, const ServerParams& P, const Job& J, uint64_t t, uint32_t sh) {
  const uint64_t A = J.out_start >> sh;
  const uint64_t a = max(J.out_start, (A + t) << sh), b = min(J.out_end, (A + t + 1) << sh);
  if (J.type == JOB_DEC) {
    DecCtx c;
    dec_ctx_init(c, P.ix, J, P.rings[J.out_ring]);  // (base and mask: the decode reads no cursor from it)
    dec_tile_generic(T, c, a, b, 0);
  } else if (J.type == JOB_ENC) {
    EncCtx c;
    enc_ctx_init(c, P.sc, J, P.send[J.out_ring], P.sc.pieces + J.piece0);
    enc_tile_generic(T, c, a - J.out_start, b - J.out_start);
  }
}

// ---- lean steps ----------------------------------------------------------------------------------------------
// The common small step -- a few well-formed memcpy CALLs (RFC 5531 §9 call with AUTH_NONE credential and
// verifier, one record-marking fragment each, the built-in HtoD / DtoH schemas), every one of them served OK --
// done by one warp over a shared-memory copy of the windows, with no table round trips between the phases:
// lane 0 walks the header chains, lane k checks record k and makes its serve decision, a warp scan gives the reply
// offsets; then the whole CTA writes the index tables (exactly what the general phases write for such a step),
// copies the HtoD payloads and encodes the replies.  Every check of the general path is evaluated; a step that
// fails any of them (an incomplete or malformed record, another procedure, a duplicate xid, a status other than
// OK, a window or reply too large for the CTA) is left untouched -- nothing global has been written -- and runs
// through the general phases, whose first failing check is then the oracle's.
//
// The code is kept small on purpose (loops not unrolled, the word reader out of line): a one-CTA kernel runs
// instruction-fetch bound once its path leaves the 32 KB instruction cache (B300_MICROARCH.md "I-cache"), which
// is where the general phases' time goes.
constexpr uint32_t kLeanWin = 64 * 1024;   // shadow bytes (the server's dynamic shared memory)
constexpr uint32_t kLeanRecs = 32;          // records: one per lane of warp 0
constexpr uint32_t kLeanRings = 8;
constexpr uint64_t kLeanD2H = 64 * 1024;    // DtoH reply data the CTA encodes itself

struct LeanRec {
  uint64_t cur, ptr, n, off, c, size;  // header cursor; HtoD dst / DtoH src; bytes copied / DtoH size; reply cursor;
                                       // HtoD opaque count and size argument
  uint32_t len, ring, slot, xid, d2h, Ll, w, so_, sm_, pad_;
};
struct LeanState {
  LeanRec rec[kLeanRecs];
  uint32_t prefix[kLeanRings + 1];
  uint32_t soff[kLeanRings], smask[kLeanRings];
  uint64_t reply_bytes[kLeanRings];
  uint32_t ok;
};

__device__ __forceinline__ uint32_t pow2_at_least(uint64_t x) {  // >= 256
  return x <= 256 ? 256u : 1u << (32 - __clz((uint32_t)(x - 1)));
}

// Big-endian word at cursor c of a shadow ring (any alignment, across the shadow's wrap).
__device__ __noinline__ uint32_t shadow_be32(const uint8_t* sh, uint32_t so, uint32_t sm, uint64_t c) {
  const uint32_t o = (uint32_t)(c & sm);
  if (!(o & 3)) return bswap32(*reinterpret_cast<const uint32_t*>(sh + so + o));  // an aligned word (shadows are
  uint32_t v = 0;                                                                  // 256-byte aligned, >= 256 B)
#pragma unroll 1
  for (uint32_t k = 0; k < 4; ++k) v = (v << 8) | sh[so + ((c + k) & sm)];
  return v;
}

__device__ __noinline__ bool region_ok(const ServerParams& P, uint64_t ptr, uint64_t n) {
  return ptr >= P.region_base && n <= P.region_bytes && ptr - P.region_base <= P.region_bytes - n;
}

// Returns true when the step was served here (tables, payloads, replies, the bell's results); false leaves every
// global location as it was for the general phases.  Uniform across the CTA.
__device__ bool lean_step(const ServerParams& P, const SchemaTable& sch, const uint64_t* head, const uint64_t* tail,
                          const uint64_t* soff_bell, uint8_t* sh, LeanState& L, crk_server_bell* B) {
  const uint32_t n = P.n_rings, tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const IndexDev& ix = P.ix;
  const ConfigDev& cfg = P.cfg;
  if (n > kLeanRings || (cfg.F & 3) || cfg.F == 0) return false;
  // ---- the windows' shadow layout (thread 0) and their copy into shared memory (every thread)
  if (tid == 0) {
    uint32_t so = 0, ok = 1;
#pragma unroll 1
    for (uint32_t r = 0; r < n; ++r) {
      const uint64_t span = ((tail[r] + 15) & ~15ull) - (head[r] & ~15ull);
      const uint32_t c = pow2_at_least(span);
      if (tail[r] < head[r] || tail[r] - head[r] > P.rings[r].mask + 1 || span > kLeanWin) ok = 0;  // bad window
      L.soff[r] = so;
      L.smask[r] = c - 1;
      so += ok ? c : 0;
    }
    L.ok = ok && so <= kLeanWin;
  }
  cta_barrier();
  if (!L.ok) return false;
#pragma unroll 1
  for (uint32_t r = 0; r < n; ++r) {
    const uint64_t a = head[r] & ~15ull;
    const uint32_t nch = (uint32_t)((((tail[r] + 15) & ~15ull) - a) >> 4);
    const RingDesc R = P.rings[r];
#pragma unroll 1
    for (uint32_t i = tid; i < nch; i += blockDim.x) {
      const uint64_t cur = a + 16ull * i;
      *reinterpret_cast<uint4*>(sh + L.soff[r] + (uint32_t)(cur & L.smask[r])) = ld16_stream(R.base + (cur & R.mask));
    }
  }
  cta_barrier();
  STEP_MARK(tid == 0, 21, 0);
  // ---- warp 0: the chains, the records' checks and serve decisions, the reply offsets
  if (warp == 0) {
    uint32_t ok = 1, nrec = 0;
    if (lane == 0) {  // RFC 5531 §11 chains: every header a whole record (last bit), each record inside the window
#pragma unroll 1
      for (uint32_t r = 0; r < n; ++r) {
        L.prefix[r] = nrec;
        uint64_t p = head[r];
        uint32_t nr = 0;
#pragma unroll 1
        while (ok && p < tail[r]) {
          const uint32_t h = p + 4 <= tail[r] ? shadow_be32(sh, L.soff[r], L.smask[r], p) : 0u, len = h & 0x7fffffffu;
          if (!(h >> 31) || len < 40 || p + 4 + len > tail[r] || len > cfg.max_record_bytes || nrec >= kLeanRecs ||
              nr >= ix.recs_per_ring || nr >= ix.frags_per_ring) { ok = 0; break; }
          LeanRec& q = L.rec[nrec++];
          q.cur = p;
          q.len = len;
          q.ring = r;
          q.slot = nr++;
          q.so_ = L.soff[r];
          q.sm_ = L.smask[r];
          p += 4 + len;
        }
      }
      L.prefix[n] = nrec;
      STEP_MARK(true, 22, nrec);
    }
    ok = __shfl_sync(0xffffffffu, ok, 0);
    nrec = __shfl_sync(0xffffffffu, nrec, 0);
    __syncwarp();
    bool good = true;
    uint32_t xid = lane, ring = 0, w = 0;
    uint64_t d2h_bytes = 0;
    if (ok && lane < nrec) {
      LeanRec& q = L.rec[lane];
      ring = q.ring;
      const uint64_t b0 = q.cur + 4;  // logical offset 0
      uint32_t wv[14];                // the fixed-layout head (and the DtoH arguments)
      const uint32_t o0 = (uint32_t)(b0 & q.sm_);
      if (!(o0 & 3) && o0 + 56 <= q.sm_ + 1) {  // aligned and not across the shadow's wrap: 14 independent loads
        const uint32_t* wp = reinterpret_cast<const uint32_t*>(sh + q.so_ + o0);
#pragma unroll
        for (uint32_t k = 0; k < 14; ++k) wv[k] = bswap32(wp[k]);
      } else {
#pragma unroll 1
        for (uint32_t k = 0; k < 14; ++k) wv[k] = shadow_be32(sh, q.so_, q.sm_, b0 + 4 * k);
      }
      xid = wv[0];
      // RFC 5531 §9: CALL, rpcvers 2, the program and version, zero-length credential and verifier bodies
      good = wv[1] == 0 && wv[2] == 2 && wv[3] == cfg.prog && wv[4] == cfg.vers && wv[7] == 0 && wv[9] == 0;
      const uint32_t proc = wv[5];
      uint32_t e = 0;  // the procedure's first schema entry must be the built-in memcpy layout
#pragma unroll 1
      while (e < sch.n && sch.s[e].proc != proc) ++e;
      const Schema* s = e < sch.n ? &sch.s[e] : nullptr;
      const bool h2d = good && s && proc == cfg.proc_h2d && s->n_items == 3 && s->items[0] == CRK_K_U64 &&
                       s->items[1] == CRK_K_OPAQUE_VAR && s->items[2] == CRK_K_U64;
      const bool d2h = good && s && proc == cfg.proc_d2h && s->n_items == 2 && s->items[0] == CRK_K_U64 &&
                       s->items[1] == CRK_K_U64;
      q.ptr = ((uint64_t)wv[10] << 32) | wv[11];
      q.d2h = d2h;
      good = h2d || d2h;
      if (h2d) {  // RFC 4506 §4.10 opaque<>: count, bytes, zero pad; then the size hyper; nothing after it
        const uint64_t c = wv[12], pn = pad4(c), o2 = 52 + c + pn;
        good = o2 + 8 == q.len;
#pragma unroll 1
        for (uint64_t i = 0; good && cfg.strict && i < pn; ++i) good = sh[q.so_ + ((b0 + 52 + c + i) & q.sm_)] == 0;
        const uint64_t size = good ? ((uint64_t)shadow_be32(sh, q.so_, q.sm_, b0 + o2) << 32) |
                                         shadow_be32(sh, q.so_, q.sm_, b0 + o2 + 4) : 0;
        good = good && !(cfg.strict && c != size);              // E_SIZE (reading R9)
        q.c = c;
        q.size = size;
        q.n = (cfg.strict || c <= size) ? c : size;
        good = good && region_ok(P, q.ptr, q.n);                // E_PTR
        q.Ll = 28;
      } else if (d2h) {
        q.n = ((uint64_t)wv[12] << 32) | wv[13];
        good = q.len == 56 && q.n <= 0xffffffffull && region_ok(P, q.ptr, q.n);  // E_PTR (reading R21)
        d2h_bytes = q.n;
        q.Ll = (uint32_t)(32 + q.n + pad4(q.n));
      }
      w = good ? (uint32_t)wire_of(q.Ll, cfg.F) : 0;
      q.w = w;
      q.xid = xid;
      good = good && !(soff_bell[ring] & 3);  // replies are written as aligned words
    }
    STEP_MARK(lane == 0, 23, w);
    // xids distinct (reading R11: a repeated xid is E_XID for the later record)
#pragma unroll 1
    for (uint32_t j = 1; j < nrec; ++j) {  // (nrec is warp-uniform)
      const uint32_t xj = __shfl_sync(0xffffffffu, xid, j - 1);
      if (j - 1 < lane && lane < nrec && xj == xid) good = false;
    }
    uint64_t tot = d2h_bytes, incl = lane < nrec ? w : 0;
#pragma unroll 1
    for (uint32_t o = 1; o < 32; o <<= 1) {
      tot += __shfl_xor_sync(0xffffffffu, tot, o);
      const uint64_t y = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += y;
    }
    ok = ok && !__any_sync(0xffffffffu, lane < nrec && !good) && tot <= kLeanD2H;
    // reply cursors: per ring, the exclusive prefix of the wire sizes in record order
    const uint64_t excl = incl - (lane < nrec ? w : 0);
    const uint32_t first = ok && lane < nrec ? L.prefix[ring] : 0;
    const uint64_t ring0 = __shfl_sync(0xffffffffu, excl, first & 31);
    if (ok && lane < nrec) {
      L.rec[lane].off = soff_bell[ring] + (excl - ring0);
      if (lane + 1 == L.prefix[ring + 1]) L.reply_bytes[ring] = incl - ring0;  // the ring's last record
    }
    if (ok && lane < n && L.prefix[lane + 1] == L.prefix[lane]) L.reply_bytes[lane] = 0;
    if (lane == 0) L.ok = ok;
    STEP_MARK(lane == 0, 24, ok);
  }
  cta_barrier();
  if (!L.ok) return false;
  STEP_MARK(tid == 0, 25, 0);
  // ---- the index tables (what the general scan / parse / plan write for this step) and the results
  const uint32_t N = L.prefix[n], FC = ix.frags_per_ring, RC = ix.recs_per_ring;
  if (tid < n) {
    RingDesc R = P.rings[tid];
    R.head = head[tid];
    R.tail = tail[tid];
    ix.rings[tid] = R;
    crk_ring_result rr;
    rr.status = CRK_OK;
    rr.n_records = rr.n_frags = L.prefix[tid + 1] - L.prefix[tid];
    rr.rec_base = L.prefix[tid];
    rr.consumed = tail[tid];
    rr.reply_bytes = L.reply_bytes[tid];
    ix.res[tid] = rr;
    B->res[tid] = rr;
    ix.rec_prefix[tid] = L.prefix[tid];
  }
  if (tid == 0) {
    ix.rec_prefix[n] = N;
    *ix.total = N;
    B->status = CRK_OK;
  }
  if (tid < N) {
    const LeanRec& q = L.rec[tid];
    const uint32_t d = tid, fs = q.ring * FC + q.slot, rs = q.ring * RC + q.slot;
    ix.frag_phys[fs] = q.cur + 4;
    ix.frag_lstart[fs] = 0;
    ix.frag_hdr[fs] = q.len | 0x80000000u;
    ix.rec_begin[rs] = q.cur;
    ix.rec_len[rs] = q.len;
    ix.rec_frag0[rs] = fs;
    ix.rec_nfrags[rs] = 1;
    ix.p_slot[d] = rs;
    ix.p_ring[d] = q.ring;
    ix.p_xid[d] = q.xid;
    ix.p_proc[d] = q.d2h ? cfg.proc_d2h : cfg.proc_h2d;
    ix.p_status[d] = CRK_OK;
    ix.p_nitems[d] = q.d2h ? 2 : 3;
    ix.p_frag0[d] = fs;
    ix.p_nfrags[d] = 1;
    ix.p_flen0[d] = q.len;
    // items: u64 ptr @40; then DtoH: u64 size @48; HtoD: opaque<> @52 (count c), u64 size after its pad
    const uint64_t b = (uint64_t)d * kMaxItems, o2 = 52 + q.c + pad4(q.c), size = q.d2h ? q.n : q.size;
    ix.p_kind[b] = CRK_K_U64;
    ix.p_off[b] = 40;
    ix.p_count[b] = 0;
    ix.p_value[b] = q.ptr;
    ix.p_kind[b + 1] = q.d2h ? CRK_K_U64 : CRK_K_OPAQUE_VAR;
    ix.p_off[b + 1] = q.d2h ? 48 : 52;
    ix.p_count[b + 1] = q.d2h ? 0 : q.c;
    ix.p_value[b + 1] = q.d2h ? size : 0;
    if (!q.d2h) {
      ix.p_kind[b + 2] = CRK_K_U64;
      ix.p_off[b + 2] = o2;
      ix.p_count[b + 2] = 0;
      ix.p_value[b + 2] = size;
    }
    ix.s_status[d] = CRK_OK;
    ix.s_reply_err[d] = 0;
    ix.s_reply_off[d] = q.off;
    ix.s_reply_wire[d] = q.w;
    // distinct xids into the cleared table: the first free slot (a lone record's is its home slot: a plain store)
    const unsigned long long key = ((unsigned long long)q.xid << 32) | d;
    uint32_t h = (q.xid * 0x9E3779B1u) & ix.hash_mask;
    if (N == 1) ix.xid_hash[h] = key;
    else
#pragma unroll 1
      for (;; h = (h + 1) & ix.hash_mask)
        if (atomicCAS(ix.xid_hash + h, ~0ull, key) == ~0ull) break;
  }
  STEP_MARK(tid == 0, 26, 0);
  // ---- HtoD payloads (shadow -> destination) and the framed replies (aligned words into the send rings)
#pragma unroll 1
  for (uint32_t d = 0; d < N; ++d) {
    const LeanRec& q = L.rec[d];
    if (!q.d2h) {
      uint8_t* dst = reinterpret_cast<uint8_t*>(q.ptr);
#pragma unroll 1
      for (uint64_t i = tid; i < q.n; i += blockDim.x) dst[i] = sh[q.so_ + ((q.cur + 56 + i) & q.sm_)];
    }
    const RingDesc O = P.send[q.ring];
    const uint8_t* src = reinterpret_cast<const uint8_t*>(q.ptr);
    const uint32_t F = cfg.F;
#pragma unroll 1
    for (uint32_t k = tid; k < (q.w >> 2); k += blockDim.x) {
      const uint32_t pos = 4 * k, f = pos / (F + 4), within = pos - f * (F + 4);
      uint32_t v;
      if (within == 0) {  // RFC 5531 §11 fragment header
        const uint32_t flen = min(F, q.Ll - f * F);
        v = flen | ((f * F + flen == q.Ll) ? 0x80000000u : 0u);
      } else {  // REPLY: xid, REPLY 1, MSG_ACCEPTED 0, AUTH_NONE 0 / 0, SUCCESS 0, err 0, [DtoH: n, data, pad]
        const uint32_t l0 = f * F + within - 4;
        if (l0 < (q.d2h ? 32u : 28u)) {
          v = l0 == 0 ? q.xid : l0 == 4 ? 1u : l0 == 28 ? (uint32_t)q.n : 0u;
        } else {
          v = 0;
#pragma unroll 1
          for (uint32_t j = 0; j < 4; ++j) {
            const uint64_t di = l0 + j - 32;
            v = (v << 8) | (di < q.n ? src[di] : 0u);
          }
        }
      }
      *reinterpret_cast<uint32_t*>(O.base + ((q.off + pos) & O.mask)) = bswap32(v);
    }
  }
  STEP_MARK(tid == 0, 31, 0);
  cta_barrier();
  return true;
}

__global__ void __launch_bounds__(kServerThreads, 1) server_kernel(ServerParams P) {
  extern __shared__ __align__(16) uint8_t lean_sh[];  // kLeanWin: the windows of a lean step
  __shared__ LeanState lean_s;
  __shared__ ScanState S;
  __shared__ SchemaTable sch;
  __shared__ __align__(16) uint8_t heads[kServerWarps][kHeadBuf];
  __shared__ SendRingsParam send;
  __shared__ uint64_t warp_sums[32];
  __shared__ uint64_t ring_first_pre[kMaxRings];
  __shared__ uint32_t prefix[kMaxRings + 1];
  __shared__ uint64_t win_head[kMaxRings], win_tail[kMaxRings];
  __shared__ uint64_t seq_s;
  __shared__ Job jobs_s[kJobCache];
  __shared__ uint64_t tiles_s, reply_s[kMaxRings];
  __shared__ crk_ring_result res_s[kMaxRings];
  __shared__ uint32_t stop_s, bad_s;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  crk_server_bell* B = P.bell;
  const IndexDev& ix = P.ix;
  uint64_t seen = B->done_seq;
  if (threadIdx.x == 0) seq_s = seen;
  cta_barrier();
  for (;;) {
    // ---- wait for a new step: lane 0 of kPollers warps polls the doorbell (one read in flight each; more than
    // one poller measured slower: their reads contend on the link)
    if (lane == 0 && warp < kPollers) {
      uint64_t s;
      while ((s = ld_acquire_sys(&B->seq)) == seen && *(volatile uint64_t*)&seq_s == seen) __nanosleep(64 + 96 * warp);
      if (s != seen) seq_s = s;  // every poller that saw it stores the same value
    }
    phase_sync();
    // the stop flag is read with the step's cursors (one round trip) and checked after the setup barrier
    if (threadIdx.x == 0) {
      bad_s = 0;
      B->t_begin_ns = gtimer();
    }
    TL_END(P.cfg, 6);
    seen = seq_s;
    // ---- step setup: schemas (re-read: registrations may follow the start), send cursors, xid table
    for (uint32_t i = threadIdx.x; i < sizeof(SchemaTable) / 4; i += blockDim.x)
      reinterpret_cast<uint32_t*>(&sch)[i] = reinterpret_cast<const uint32_t*>(P.schemas)[i];
    // the step's cursors: one read of the bell per value, all in flight at once (a host bell is read
    // over PCIe; every later use is from shared memory)
    if (threadIdx.x == blockDim.x - 1) stop_s = *(volatile uint64_t*)&B->stop != 0;
    for (uint32_t r = threadIdx.x; r < P.n_rings; r += blockDim.x) {
      send.r[r] = P.send[r];
      send.off[r] = *(volatile uint64_t*)&B->send_off[r];
      win_head[r] = *(volatile uint64_t*)&B->head[r];
      win_tail[r] = *(volatile uint64_t*)&B->tail[r];
    }
    if (threadIdx.x == 0) {
      send.n_rings = P.n_rings;
      send.doorbell = nullptr;
    }
    for (uint64_t h = threadIdx.x; h <= ix.hash_mask; h += blockDim.x) ix.xid_hash[h] = ~0ull;
    phase_sync();
    if (stop_s) break;
    TL_END(P.cfg, 0);
    if (threadIdx.x == 0) B->t_phase_ns[0] = gtimer();
    STEP_MARK(threadIdx.x == 0, 0, 0);
    // ---- a lean step (well-formed memcpy CALLs only), else the general phases
    if (lean_step(P, sch, win_head, win_tail, send.off, lean_sh, lean_s, B)) {
      if (threadIdx.x == 0) {
        const uint64_t t = gtimer();
        for (int k = 1; k < 5; ++k) B->t_phase_ns[k] = t;
      }
    } else {
    // ---- K1: each ring in turn by the whole CTA
    SCAN_TRACE(threadIdx.x == 0, 5, 0);
    if (threadIdx.x == 0) prefix[0] = 0;
    for (uint32_t r = 0; r < P.n_rings; ++r) {
      RingDesc R = P.rings[r];
      R.head = win_head[r];
      R.tail = win_tail[r];
      const bool bad = R.tail < R.head || R.tail - R.head > R.mask + 1;
      if (bad) {
        R.tail = R.head;
        if (threadIdx.x == 0) bad_s = 1;
      }
      scan_ring_cta(ix, R, bad, r, P.cfg, S);
      if (threadIdx.x == 0) prefix[r + 1] = prefix[r] + S.nr;
    }
    if (threadIdx.x == 0) dense_numbering_cta(ix, P.n_rings, prefix);
    phase_sync();
    TL_END(P.cfg, 1);
    if (threadIdx.x == 0) B->t_phase_ns[1] = gtimer();
#ifdef CRK_TIMELINE_SCAN2  // diagnostic: the scan again, with its code and data now cached
    for (uint32_t r = 0; r < P.n_rings; ++r) {
      RingDesc R = P.rings[r];
      R.head = win_head[r];
      R.tail = win_tail[r];
      const bool bad = R.tail < R.head || R.tail - R.head > R.mask + 1;
      if (bad) R.tail = R.head;
      scan_ring_cta(ix, R, bad, r, P.cfg, S);
      if (threadIdx.x == 0) prefix[r + 1] = prefix[r] + S.nr;
    }
    if (threadIdx.x == 0) dense_numbering_cta(ix, P.n_rings, prefix);
    phase_sync();
    TL_END(P.cfg, 7);
#endif
    // the rings' scan results (final but for reply_bytes, which the plan hands over in shared memory): copied to
    // shared memory now by the last warp (the first parses record 0), overlapping the parse
    if (warp == kServerWarps - 1)
      for (uint32_t r = lane; r < P.n_rings; r += 32) {
        res_s[r] = ix.res[r];
        reply_s[r] = 0;
      }
    // ---- K3: one warp per record (prefix[] is the scan's dense numbering, in shared memory)
    const uint32_t total = prefix[P.n_rings];
    for (uint32_t d = warp; d < total; d += kServerWarps) {
      uint32_t lo = 0, hi = P.n_rings;  // ring of dense record d
      while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (prefix[mid] <= d) lo = mid; else hi = mid;
      }
      parse_record(ix, sch, P.cfg, d, lo, lo * ix.recs_per_ring + (d - prefix[lo]), heads[warp], lane, total == 1,
                   (P.dev_rings >> lo) & 1 ? kPrefetchMax : 0);
      __syncwarp();
    }
    phase_sync();
    TL_END(P.cfg, 2);
    if (threadIdx.x == 0) B->t_phase_ns[2] = gtimer();
    // ---- serve planning (statuses, reply offsets, jobs)
    const PlanOut out{jobs_s, kJobCache, &tiles_s, reply_s};
    plan_small_block(ix, P.cfg, P.sc, send, P.region_base, P.region_bytes, warp_sums, ring_first_pre, prefix, &out);
    phase_sync();
    TL_END(P.cfg, 3);
    if (threadIdx.x == 0) B->t_phase_ns[3] = gtimer();
    // ---- movers: every job cut into 8 KiB output tiles, tiles dealt to the warps round-robin
    const uint32_t n_jobs = 2 * total;
    const Team TW{lane, 32, 0, 1};
    // the plan's tile total and (up to kJobCache) jobs are in shared memory; more jobs are read from the scratch
    const uint64_t plan_tiles = tiles_s;
    if (n_jobs > kJobCache) {  // the first kJobCache jobs in one round trip (every warp walks every descriptor)
      for (uint32_t i = threadIdx.x; i < kJobCache * (uint32_t)(sizeof(Job) / 4); i += blockDim.x)
        reinterpret_cast<uint32_t*>(jobs_s)[i] = reinterpret_cast<const uint32_t*>(P.sc.jobs)[i];
      cta_barrier();
    }
    // the results go to the bell now (host-memory writes in flight during the move; the release after the
    // move orders them before done_seq)
    if (threadIdx.x < P.n_rings) {
      crk_ring_result my_res = res_s[threadIdx.x];
      my_res.reply_bytes = reply_s[threadIdx.x];
      B->res[threadIdx.x] = my_res;
    }
    if (threadIdx.x == 0) B->status = bad_s ? CRK_E_ARG : CRK_OK;
    const uint32_t sh = plan_tiles <= 4 ? 11u : 13u;
    STEP_MARK(threadIdx.x == 0, 16, sh ^ jobs_s[0].type);
    uint64_t first = 0;  // global number of the job's first tile
    for (uint32_t j = 0; j < n_jobs; ++j) {
      const Job J = j < kJobCache ? jobs_s[j] : P.sc.jobs[j];
      const uint64_t nt = job_tiles(J, sh);
      for (uint64_t t = (warp + kServerWarps - first % kServerWarps) % kServerWarps; t < nt; t += kServerWarps)
        move_tile(TW, P, J, t, sh);
      first += nt;
    }
    STEP_MARK(lane == 0 && warp < 4, 27 + warp, 0);  // each of the first warps' last tile done
    STEP_MARK(threadIdx.x == 0, 17, 0);
    phase_sync();
    STEP_MARK(threadIdx.x == 0, 18, 0);
    TL_END(P.cfg, 4);
    if (threadIdx.x == 0) B->t_phase_ns[4] = gtimer();
    }  // general phases
    // ---- publish: done_seq (the results were written before the move)
    cta_barrier();
    STEP_MARK(threadIdx.x == 0, 19, 0);
    if (threadIdx.x == 0) {
      B->t_end_ns = gtimer();
      // a system-scope release: the step's writes (every thread's, ordered before it by the barrier; the
      // PTX memory model's causality order is cumulative) are visible to whoever acquires done_seq
      st_release_sys(&B->done_seq, seen);
      STEP_MARK(true, 20, 0);
    }
    TL_END(P.cfg, 5);
  }
}

}  // namespace

uint32_t server_threads() { return kServerThreads; }

#ifdef CRK_SCAN_TRACE
// Diagnostic build only: the server translation unit's copy of the scan clock trace (k_scan.cuh).
extern "C" int crk_debug_server_scan_trace(unsigned long long* out, uint32_t* counts, int reset) {
  if (out && cudaMemcpyFromSymbol(out, g_scan_trace, sizeof(g_scan_trace)) != cudaSuccess) return -100;
  if (counts && cudaMemcpyFromSymbol(counts, g_scan_trace_n, sizeof(g_scan_trace_n)) != cudaSuccess) return -100;
  if (reset) {
    static const uint32_t zero[kTraceRings] = {};
    if (cudaMemcpyToSymbol(g_scan_trace_n, zero, sizeof(zero)) != cudaSuccess) return -100;
  }
  return 0;
}
#endif

#ifdef CRK_STEP_TRACE
extern "C" int crk_debug_server_step_trace(unsigned long long* out32) {
  return cudaMemcpyFromSymbol(out32, g_step_trace, sizeof(g_step_trace)) == cudaSuccess ? 0 : -100;
}
#endif

#ifdef CRK_PLAN_TRACE
extern "C" int crk_debug_server_plan_trace(unsigned long long* out16) {
  return cudaMemcpyFromSymbol(out16, g_plan_trace, sizeof(g_plan_trace)) == cudaSuccess ? 0 : -100;
}
#endif

cudaError_t launch_server(const IndexDev& ix, const ConfigDev& cfg, const Scratch& sc, const SchemaTable* schemas,
                          crk_server_bell* bell, uint32_t n_rings, const crk_ring* rings, const crk_ring* send_rings,
                          uint64_t region_base, uint64_t region_bytes, cudaStream_t s) {
  ServerParams P;
  memset(&P, 0, sizeof(P));
  P.ix = ix;
  P.cfg = cfg;
  P.sc = sc;
  P.schemas = schemas;
  P.bell = bell;
  P.n_rings = n_rings;
  for (uint32_t r = 0; r < n_rings; ++r) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, rings[r].base) == cudaSuccess && a.type == cudaMemoryTypeDevice)
      P.dev_rings |= 1ull << r;
    else
      (void)cudaGetLastError();
    P.rings[r].base = rings[r].base;
    P.rings[r].mask = rings[r].cap - 1;
    P.send[r].base = send_rings[r].base;
    P.send[r].mask = send_rings[r].cap - 1;
  }
  P.region_base = region_base;
  P.region_bytes = region_bytes;
  const cudaError_t ea = cudaFuncSetAttribute(server_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kLeanWin);
  if (ea != cudaSuccess) return ea;
  server_kernel<<<1, kServerThreads, kLeanWin, s>>>(P);
  count_launch();
  return cudaGetLastError();
}

}  // namespace crk
