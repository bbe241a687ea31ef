// K2: single-pass device-wide exclusive prefix sum (decoupled look-back).  Turns per-item sizes into
// scatter offsets: mover tiles per job, reply wire sizes -> send-ring cursors, explicit fragment
// lengths -> fragment wire starts.  The count may live on the device (set by an earlier kernel).
#include "crk_device.cuh"

namespace crk {

namespace {

constexpr int kScanBlock = 256;
constexpr int kScanIPT = 8;  // items per thread
constexpr unsigned long long kFlagAgg = 1ull << 62, kFlagInc = 2ull << 62, kValMask = (1ull << 62) - 1;

__device__ __forceinline__ unsigned long long ld_volatile(const unsigned long long* p) {
  return *reinterpret_cast<const volatile unsigned long long*>(p);
}
__device__ __forceinline__ void st_volatile(unsigned long long* p, unsigned long long v) {
  *reinterpret_cast<volatile unsigned long long*>(p) = v;
}

template <typename T>
__global__ void __launch_bounds__(kScanBlock) scan_kernel(T* data, uint32_t n_static, const uint32_t* n_dev, T* total,
                                                          unsigned long long* state, uint32_t* block_counter,
                                                          uint32_t single) {
  pdl_entry();
  __shared__ uint32_t s_bid;
  __shared__ uint64_t s_warp[kScanBlock / 32];
  __shared__ uint64_t s_excl;
  if (threadIdx.x == 0) s_bid = single ? 0u : atomicAdd(block_counter, 1u);  // launch-order ids: forward progress
  __syncthreads();
  const uint32_t bid = s_bid;
  const uint32_t n = n_dev ? *n_dev : n_static;
  const uint64_t base = (uint64_t)bid * kScanBlock * kScanIPT;
  if (base >= n && !(n == 0 && bid == 0)) return;
  uint64_t v[kScanIPT];
  uint64_t tsum = 0;
  const uint64_t my = base + (uint64_t)threadIdx.x * kScanIPT;
#pragma unroll
  for (int i = 0; i < kScanIPT; ++i) {
    v[i] = (my + i < n) ? (uint64_t)data[my + i] : 0;
    tsum += v[i];
  }
  // block exclusive scan of the per-thread sums (warp shuffles, then the warp totals)
  const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint64_t x = tsum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint64_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= (uint32_t)o) x += y;
  }
  if (lane == 31) s_warp[w] = x;
  __syncthreads();
  if (w == 0) {
    uint64_t ws = lane < kScanBlock / 32 ? s_warp[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint64_t y = __shfl_up_sync(0xffffffffu, ws, o);
      if (lane >= (uint32_t)o) ws += y;
    }
    if (lane < kScanBlock / 32) s_warp[lane] = ws;  // inclusive warp prefixes
  }
  __syncthreads();
  const uint64_t block_total = s_warp[kScanBlock / 32 - 1];
  const uint64_t thread_excl = x - tsum + (w ? s_warp[w - 1] : 0);
  if (threadIdx.x == 0) {
    uint64_t excl = 0;
    if (bid == 0) {
      if (!single) st_volatile(state, kFlagInc | (block_total & kValMask));
    } else {
      st_volatile(state + bid, kFlagAgg | (block_total & kValMask));
      int64_t j = (int64_t)bid - 1;
      for (;;) {
        unsigned long long s = ld_volatile(state + j);
        if ((s >> 62) == 0) continue;  // predecessor not published yet
        excl += s & kValMask;
        if ((s >> 62) == 2) break;
        --j;
      }
      st_volatile(state + bid, kFlagInc | ((excl + block_total) & kValMask));
    }
    s_excl = excl;
  }
  __syncthreads();
  uint64_t run = s_excl + thread_excl;
#pragma unroll
  for (int i = 0; i < kScanIPT; ++i) {
    if (my + i < n) data[my + i] = (T)run;
    run += v[i];
  }
  if (total && (base + (uint64_t)kScanBlock * kScanIPT >= n) && threadIdx.x == 0) *total = (T)(s_excl + block_total);
}

template <typename T>
cudaError_t launch_scan(T* data, uint32_t n, const uint32_t* n_dev, T* total, Scratch& sc, cudaStream_t s) {
  // n is the (host-known) upper bound when n_dev is given
  const uint32_t per = kScanBlock * kScanIPT;
  const uint32_t blocks = n == 0 ? 1 : (n + per - 1) / per;
  if (blocks == 1) {  // one block: no look-back, no state to reset
    CRK_LAUNCH(sc.pdl != 0, scan_kernel<T>, 1, kScanBlock, 0, s, data, n, n_dev, total, sc.scan_state, sc.counters + 5, 1u);
    return cudaGetLastError();
  }
  cudaError_t e = cudaMemsetAsync(sc.scan_state, 0, sizeof(unsigned long long) * (blocks + 1), s);
  if (e != cudaSuccess) return e;
  e = cudaMemsetAsync(sc.counters + 5, 0, sizeof(uint32_t), s);
  if (e != cudaSuccess) return e;
  CRK_LAUNCH(sc.pdl != 0, scan_kernel<T>, blocks, kScanBlock, 0, s, data, n, n_dev, total, sc.scan_state, sc.counters + 5, 0u);
  return cudaGetLastError();
}

}  // namespace

cudaError_t launch_exclusive_scan_u64(uint64_t* data, uint32_t n, const uint32_t* n_dev, uint64_t* total, Scratch& sc,
                                      cudaStream_t s) {
  return launch_scan<uint64_t>(data, n, n_dev, total, sc, s);
}
cudaError_t launch_exclusive_scan_u32(uint32_t* data, uint32_t n, const uint32_t* n_dev, uint32_t* total, Scratch& sc,
                                      cudaStream_t s) {
  return launch_scan<uint32_t>(data, n, n_dev, total, sc, s);
}

}  // namespace crk
