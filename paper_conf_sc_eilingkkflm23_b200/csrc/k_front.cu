// Fused front end for small steps: K1 (scan), K3 (parse) and the one-block serve planner in ONE launch
// of one CTA, followed by the ordinary mover launch (crk_serve); scan + parse only for a small
// crk_rpc_frame_scan.  A small step (a few records, e.g. one forwarded cudaMemcpy of a few KiB: SURVEY.md
// §8(d) C1 and the small end of the C3 sweep) is a chain of dependent memory round trips; as five
// launches (hash clear, scan, parse, plan, mover) each round trip also pays a launch gap.  The device
// functions are the launched kernels' own (scan_ring_cta, parse_record, plan_small_block), so the index
// tables, statuses and jobs are identical; the phases hand data to each other inside the CTA, ordered by
// block barriers.
//
// A step of well-formed single-fragment memcpy CALLs takes the lean path (k_lean.cuh): one warp over a shared-
// memory copy of the windows, the CTA moving the payloads and replies itself, an empty plan left for the mover.
#include <mutex>

#include "k_lean.cuh"
#include "k_parse.cuh"
#include "k_plan.cuh"
#include "k_scan.cuh"

namespace crk {

namespace {

constexpr uint32_t kFrontThreads = kSmallServe;  // plan_small_block: thread d owns record d
constexpr uint32_t kFrontWarps = kFrontThreads / 32;

struct FrontParams {
  IndexDev ix;
  ConfigDev cfg;
  Scratch sc;
  const SchemaTable* schemas;
  ScanRingsParam rings;  // cursors in r[] or, with rings.doorbell, read here at execution time
  SendRingsParam send;
  uint64_t region_base, region_bytes;
  uint32_t plan;         // 0: scan + parse only (crk_rpc_frame_scan)
};

#ifdef CRK_FRONT_TRACE
// Diagnostic build only: %globaltimer at the fused front end's phase ends (thread 0).
__device__ unsigned long long g_front_trace[8];
#define FRONT_MARK(i) do { if (threadIdx.x == 0) { unsigned long long t_; \
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_)); g_front_trace[i] = t_; } } while (0)
#else
#define FRONT_MARK(i) do { } while (0)
#endif

__global__ void __launch_bounds__(kFrontThreads, 1) front_small_kernel(FrontParams P) {
  pdl_entry();
  extern __shared__ __align__(16) uint8_t lean_sh[];  // kLeanWin: the windows of a lean step
  __shared__ LeanState lean_s;
  __shared__ uint64_t win_head[kLeanRings], win_tail[kLeanRings], send_off[kLeanRings];
  __shared__ ScanState S;
  __shared__ SchemaTable sch;
  __shared__ __align__(16) uint8_t heads[kFrontWarps][kHeadBuf];
  __shared__ uint64_t warp_sums[32];
  __shared__ uint64_t ring_first_pre[kMaxRings];
  __shared__ uint32_t prefix[kMaxRings + 1];
  FRONT_MARK(0);
  TL_BEGIN(P.cfg, TL_FUSED);
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const IndexDev& ix = P.ix;
  const uint32_t n_rings = P.rings.n_rings;
  // ---- setup: an empty xid table (the schemas are loaded below, for the general phases only)
  for (uint64_t h = threadIdx.x; h <= ix.hash_mask; h += blockDim.x) ix.xid_hash[h] = ~0ull;
  // a serve step over at most kLeanRings rings: its cursors (doorbell or parameters) for the lean path
  // (the context's lean back-off, scratch counter 15: steps left before the lean path is tried again)
  __shared__ uint32_t lean_skip;
  if (threadIdx.x == 0) lean_skip = P.sc.counters[15];
  const bool try_lean = P.cfg.lean && P.plan && n_rings <= kLeanRings;
  if (try_lean && threadIdx.x < n_rings) {
    const uint32_t r = threadIdx.x;
    win_head[r] = P.rings.doorbell ? P.rings.doorbell[r] : P.rings.r[r].head;
    win_tail[r] = P.rings.doorbell ? P.rings.doorbell[n_rings + r] : P.rings.r[r].tail;
    send_off[r] = P.send.doorbell ? P.send.doorbell[2 * n_rings + r] : P.send.off[r];
  }
  cta_barrier();
  FRONT_MARK(1);
  if (try_lean && lean_skip == 0) {
    const LeanMover mv{P.sc.scan_tmp + P.sc.max_jobs + 1, P.sc.counters};
    if (lean_step<false>(ix, P.cfg, n_rings, [&](uint32_t r) { return P.rings.r[r]; },
                  [&](uint32_t r) { return P.send.r[r]; }, win_head, win_tail, send_off, P.region_base,
                  P.region_bytes, lean_sh, lean_s, nullptr, &mv, nullptr)) {
      TL_END(P.cfg, TL_FUSED);
      return;
    }
    if (threadIdx.x == 0) P.sc.counters[15] = P.cfg.lean_backoff;
  } else if (try_lean && threadIdx.x == 0) {
    P.sc.counters[15] = lean_skip - 1;
  }
  for (uint32_t i = threadIdx.x; i < sizeof(SchemaTable) / 4; i += blockDim.x)
    reinterpret_cast<uint32_t*>(&sch)[i] = reinterpret_cast<const uint32_t*>(P.schemas)[i];
  cta_barrier();
  // ---- K1: each ring in turn by the whole CTA, then dense record numbering (prefix[] in shared memory)
  if (threadIdx.x == 0) prefix[0] = 0;
  for (uint32_t r = 0; r < n_rings; ++r) {
    RingDesc R = P.rings.r[r];
    bool bad = false;
    if (P.rings.doorbell) {
      R.head = P.rings.doorbell[r];
      R.tail = P.rings.doorbell[n_rings + r];
      bad = R.tail < R.head || R.tail - R.head > R.mask + 1;
      if (bad) R.tail = R.head;
    }
    scan_ring_cta(ix, R, bad, r, P.cfg, S);
    if (threadIdx.x == 0) prefix[r + 1] = prefix[r] + S.nr;
  }
  if (threadIdx.x == 0) dense_numbering_cta(ix, n_rings, prefix);
  cta_barrier();
  FRONT_MARK(2);
  // ---- K3: one warp per record
  const uint32_t total = prefix[n_rings];
  for (uint32_t d = warp; d < total; d += kFrontWarps) {
    uint32_t lo = 0, hi = n_rings;  // ring of dense record d
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (prefix[mid] <= d) lo = mid; else hi = mid;
    }
    parse_record(ix, sch, P.cfg, d, lo, lo * ix.recs_per_ring + (d - prefix[lo]), heads[warp], lane, total == 1);
    __syncwarp();
  }
  if (!P.plan) {
    TL_END(P.cfg, TL_FUSED);
    return;
  }
  cta_barrier();
  FRONT_MARK(3);
  // ---- serve planning: statuses, reply offsets, jobs, their tile prefix, mover cursors
  plan_small_block(ix, P.cfg, P.sc, P.send, P.region_base, P.region_bytes, warp_sums, ring_first_pre, prefix);
  FRONT_MARK(4);
  TL_END(P.cfg, TL_FUSED);
}

}  // namespace

uint32_t front_small_threads() { return kFrontThreads; }

#ifdef CRK_FRONT_TRACE
extern "C" int crk_debug_front_trace(unsigned long long* out8) {
  return cudaMemcpyFromSymbol(out8, g_front_trace, sizeof(g_front_trace)) == cudaSuccess ? 0 : -100;
}
#endif

cudaError_t launch_front_small(const IndexDev& ix, const ConfigDev& cfg, Scratch& sc, const SchemaTable* schemas,
                               const ScanRingsParam& rings, uint32_t n_rings, const crk_ring* send_rings,
                               const uint64_t* send_offs, uint64_t region_base, uint64_t region_bytes,
                               const uint64_t* doorbell, bool plan, cudaStream_t s) {
  FrontParams P;
  memset(&P, 0, sizeof(P));
  P.ix = ix;
  P.cfg = cfg;
  P.sc = sc;
  P.schemas = schemas;
  P.rings = rings;
  P.plan = plan;
  P.send.n_rings = n_rings;
  for (uint32_t r = 0; plan && r < n_rings; ++r) {
    P.send.r[r].base = send_rings[r].base;
    P.send.r[r].mask = send_rings[r].cap - 1;
    P.send.off[r] = send_offs ? send_offs[r] : 0;
  }
  P.send.doorbell = doorbell;
  P.region_base = region_base;
  P.region_bytes = region_bytes;
  prof_mark(PROF_SCAN, true, s);
  {  // the lean path's dynamic shared memory: a per-device opt-in, raised once
    static std::mutex mu;
    static bool set[kMaxDevices] = {};
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (dev < 0 || dev >= kMaxDevices) return cudaErrorInvalidDevice;
    std::lock_guard<std::mutex> lk(mu);
    if (!set[dev]) {
      e = cudaFuncSetAttribute(front_small_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kLeanWin);
      if (e != cudaSuccess) return e;
      set[dev] = true;
    }
  }
  CRK_LAUNCH(pdl_of(cfg), front_small_kernel, 1, kFrontThreads, kLeanWin, s, P);
  prof_mark(PROF_SCAN, false, s);
  return cudaGetLastError();
}

}  // namespace crk
