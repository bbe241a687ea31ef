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
#include "k_lean.cuh"
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
  uint32_t lean_skip = 0;  // steps left before the lean path is tried again
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
    bool lean = false;  // (lean_skip is uniform across the CTA: lean_step's answer is)
    if (P.cfg.lean && lean_skip == 0) {
      lean = lean_step<true>(ix, P.cfg, P.n_rings, [&](uint32_t r) { return P.rings[r]; },
                       [&](uint32_t r) { return P.send[r]; }, win_head, win_tail, send.off, P.region_base,
                       P.region_bytes, lean_sh, lean_s, B, nullptr, &sch);
      if (!lean) lean_skip = P.cfg.lean_backoff;
    } else if (lean_skip) {
      --lean_skip;
    }
    if (lean) {
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
