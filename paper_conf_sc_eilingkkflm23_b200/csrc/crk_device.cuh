// Device helpers shared by the crk kernels: ring access, vector I/O, byte realignment, byte swaps,
// warp/block reductions.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "crk_internal.h"

namespace crk {

__device__ __forceinline__ uint32_t bswap32(uint32_t x) { return __byte_perm(x, 0, 0x0123); }

// Loads of ring bytes that stay constant for a kernel's lifetime go through the read-only path.  The
// persistent server (k_server.cu) sees rings change under it, so it defines these as coherent loads.
#ifdef CRK_COHERENT_LOADS
#define CRK_RO_LD(p) __ldcg(p)
#else
#define CRK_RO_LD(p) __ldg(p)
#endif

// Byte at ring cursor c (RFC 5531 §11 stream position), wrap at cap (reading R16).
__device__ __forceinline__ uint8_t ring_byte(const RingDesc& R, uint64_t c) { return R.base[c & R.mask]; }

// Big-endian u32 at ring cursor c (RFC 4506 §4.1), any alignment, across the wrap.
__device__ __forceinline__ uint32_t ring_be32(const RingDesc& R, uint64_t c) {
  uint64_t o = c & R.mask;
  if ((o & 3) == 0) return bswap32(*reinterpret_cast<const uint32_t*>(R.base + o));
  return ((uint32_t)R.base[o] << 24) | ((uint32_t)R.base[(c + 1) & R.mask] << 16) |
         ((uint32_t)R.base[(c + 2) & R.mask] << 8) | (uint32_t)R.base[(c + 3) & R.mask];
}

// 16-byte streaming load of an aligned chunk (read-only for the kernel's lifetime).
__device__ __forceinline__ uint4 ld16_stream(const void* p) {
  uint4 r;
#ifdef CRK_COHERENT_LOADS
  asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];"
#else
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
#endif
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ void st16(void* p, uint4 v) {
  asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}
__device__ __forceinline__ void st16_stream(void* p, uint4 v) {
  asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}

// The 16 bytes starting `sh` (0..15) bytes into the 32-byte window a:b (memory order, little-endian
// words), i.e. a funnel shift across two aligned chunks.  sh is warp-uniform in callers.
__device__ __forceinline__ uint4 funnel16(uint4 a, uint4 b, uint32_t sh) {
  const uint32_t q = sh >> 2, r = (sh & 3) * 8;
  uint32_t w0, w1, w2, w3, w4;
  switch (q) {
    case 0: w0 = a.x; w1 = a.y; w2 = a.z; w3 = a.w; w4 = b.x; break;
    case 1: w0 = a.y; w1 = a.z; w2 = a.w; w3 = b.x; w4 = b.y; break;
    case 2: w0 = a.z; w1 = a.w; w2 = b.x; w3 = b.y; w4 = b.z; break;
    default: w0 = a.w; w1 = b.x; w2 = b.y; w3 = b.z; w4 = b.w; break;
  }
  uint4 o;
  o.x = __funnelshift_r(w0, w1, r);
  o.y = __funnelshift_r(w1, w2, r);
  o.z = __funnelshift_r(w2, w3, r);
  o.w = __funnelshift_r(w3, w4, r);
  return o;
}

// Reverse the bytes of each esize-byte element of a 16-byte chunk (RFC 4506 big-endian <-> host).
__device__ __forceinline__ uint4 swap16(uint4 v, uint32_t esize) {
  if (esize == 4) {
    v.x = bswap32(v.x); v.y = bswap32(v.y); v.z = bswap32(v.z); v.w = bswap32(v.w);
  } else if (esize == 8) {
    uint32_t x = bswap32(v.y), y = bswap32(v.x), z = bswap32(v.w), w = bswap32(v.z);
    v.x = x; v.y = y; v.z = z; v.w = w;
  }
  return v;
}

__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31; }

// CTA barriers that tolerate a warp arriving diverged (barrier.sync without .aligned; __syncthreads is the
// .aligned form, undefined when a warp's lanes reach it separately).  The single-CTA step code (scan, parse,
// planning, the CTA movers) crosses phase boundaries right after lane-dependent loops (xid probes, per-lane
// fragment walks, work done by warp 0 alone), where the warp need not have reconverged.
__device__ __forceinline__ void cta_barrier() { asm volatile("barrier.sync 0;" ::: "memory"); }
__device__ __forceinline__ bool cta_barrier_or(bool p) {
  uint32_t r;
  asm volatile(
      "{\n .reg .pred q, o;\n setp.ne.u32 q, %1, 0;\n barrier.red.or.pred o, 0, q;\n selp.u32 %0, 1, 0, o;\n}\n"
      : "=r"(r)
      : "r"((uint32_t)p)
      : "memory");
  return r != 0;
}

// Programmatic dependent launch (launch_k in crk_internal.h): the first statement of every kernel of the
// library.  griddepcontrol.wait returns once the previous kernel of the stream has completed and its memory
// is visible (a no-op without the launch attribute); launch_dependents then lets the stream's next kernel be
// scheduled, so its CTAs are resident and waiting when this one ends instead of paying the launch gap.
__device__ __forceinline__ void pdl_entry() {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

// RFC 4506 §3: bytes of zero pad after n bytes of opaque / array data
__device__ __forceinline__ uint64_t pad4(uint64_t n) { return (4 - (n & 3)) & 3; }

// Diagnostic timeline (-DCRK_TIMELINE builds; tools/timeline.py): per stage, the earliest start and the
// latest end over the CTAs of a launch, from %globaltimer (ns).
enum : uint32_t { TL_SCAN = 0, TL_PARSE = 1, TL_PLAN = 2, TL_MOVE = 3, TL_FUSED = 4, TL_STAGES = 8 };
#ifdef CRK_TIMELINE
__device__ __forceinline__ unsigned long long tl_now() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define TL_BEGIN(cfg, st) \
  do { if ((cfg).tl && threadIdx.x == 0) atomicMin((cfg).tl + 2 * (st), tl_now()); } while (0)
#define TL_END(cfg, st) \
  do { if ((cfg).tl && threadIdx.x == 0) atomicMax((cfg).tl + 2 * (st) + 1, tl_now()); } while (0)
#else
#define TL_BEGIN(cfg, st) do { } while (0)
#define TL_END(cfg, st) do { } while (0)
#endif

// Diagnostic step trace (-DCRK_STEP_TRACE builds; tools/server_step_trace.py): %globaltimer at numbered points
// of one small step, taken once `dep` (a value the point waits for) is available.  One array per translation
// unit (the persistent server's is exported).
#ifdef CRK_STEP_TRACE
__device__ unsigned long long g_step_trace[32];
#define STEP_MARK(cond, i, dep) do { if (cond) { unsigned long long t_; \
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_) : "r"((uint32_t)(dep)) : "memory"); \
  g_step_trace[i] = t_; } } while (0)
#else
#define STEP_MARK(cond, i, dep) do { } while (0)
#endif

// Block-wide min of a u32 (all threads must call).  smem: >= 32 words.
__device__ __forceinline__ uint32_t block_min_u32(uint32_t v, uint32_t* smem) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = min(v, __shfl_xor_sync(0xffffffffu, v, o));
  const uint32_t w = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  __syncthreads();
  if (lane_id() == 0) smem[w] = v;
  __syncthreads();
  v = lane_id() < nw ? smem[lane_id()] : 0xffffffffu;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = min(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// ---- mbarrier / TMA 1-D bulk copy (the mover's stages, the chunked scan's landing zones)
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n"
      "WAIT_%=: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// TMA 1-D bulk copy global -> shared (16-byte aligned, multiple of 16), completes on `bar`
__device__ __forceinline__ void bulk_g2s(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(sdst)),
               "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}

}  // namespace crk
