// K1 kernel: one CTA per ring runs scan_ring_cta (k_scan.cuh); the last CTA to finish numbers the
// records densely across rings.
#include <vector>

#include "k_scan.cuh"

namespace crk {

namespace {

__global__ void __launch_bounds__(1024) frame_scan_kernel(IndexDev ix, ScanRingsParam P, ConfigDev cfg) {
  pdl_entry();
  TL_BEGIN(cfg, TL_SCAN);
  const uint32_t ring = blockIdx.x;
  RingDesc R = P.r[ring];
  bool bad_window = false;
  if (P.doorbell) {  // cursors published by the host at execution time
    R.head = P.doorbell[ring];
    R.tail = P.doorbell[P.n_rings + ring];
    bad_window = R.tail < R.head || R.tail - R.head > R.mask + 1;
    if (bad_window) R.tail = R.head;
  }
  __shared__ ScanState S;
  scan_ring_cta(ix, R, bad_window, ring, cfg, S);
  if (threadIdx.x == 0) {
    __threadfence();
    const uint32_t done = atomicAdd(ix.ticket, 1u);
    if (done == gridDim.x - 1) {  // last ring: dense record numbering
      __threadfence();
      dense_numbering(ix, gridDim.x);
      *ix.ticket = 0;
    }
  }
  TL_END(cfg, TL_SCAN);
}

}  // namespace

#ifdef CRK_SCAN_TRACE
extern "C" int crk_debug_scan_trace(unsigned long long* out, uint32_t* counts, int reset) {
  if (out && cudaMemcpyFromSymbol(out, g_scan_trace, sizeof(g_scan_trace)) != cudaSuccess) return -100;
  if (counts && cudaMemcpyFromSymbol(counts, g_scan_trace_n, sizeof(g_scan_trace_n)) != cudaSuccess) return -100;
  if (reset) {
    static const uint32_t zero[kTraceRings] = {};
    if (cudaMemcpyToSymbol(g_scan_trace_n, zero, sizeof(zero)) != cudaSuccess) return -100;
  }
  return 0;
}
#endif

// Long windows (explicit cursors) take the chunked multi-CTA scan (k_mscan.cu); short ones, and windows
// published through a doorbell at execution time, the one-CTA-per-ring scan.
cudaError_t launch_frame_scan(const IndexDev& ix, const ScanRingsParam& p, const ConfigDev& cfg, cudaStream_t s) {
  static thread_local std::vector<unsigned char> chunk_param;
  chunk_param.resize(chunk_param_bytes());
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  prof_mark(PROF_SCAN, true, s);
  cudaError_t e;
  if (!cfg.no_chunked_scan && chunk_plan(ix, p, sms, chunk_param.data())) {
    e = launch_chunk_scan(ix, chunk_param.data(), cfg, s);
  } else {
    CRK_LAUNCH(pdl_of(cfg), frame_scan_kernel, p.n_rings, cfg.scan_threads, 0, s, ix, p, cfg);
    e = cudaGetLastError();
  }
  prof_mark(PROF_SCAN, false, s);
  return e;
}

}  // namespace crk
