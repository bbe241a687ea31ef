// K3 kernel: one warp per record runs parse_record (k_parse.cuh).
#include "k_parse.cuh"

#ifndef CRK_PARSE_CTAS_PER_SM
#define CRK_PARSE_CTAS_PER_SM 8
#endif

namespace crk {

namespace {

__global__ void __launch_bounds__(kParseWarps * 32) parse_kernel(IndexDev ix, const SchemaTable* __restrict__ tab,
                                                                  ConfigDev cfg, uint32_t n_rings) {
  pdl_entry();
  __shared__ SchemaTable sch;
  __shared__ uint32_t prefix[kMaxRings + 1];
  __shared__ __align__(16) uint8_t heads[kParseWarps][kHeadBuf];
  TL_BEGIN(cfg, TL_PARSE);
  // the grid is sized by the index's capacity: CTAs past the step's record count leave before loading anything
  const uint32_t total = *ix.total;
  if (blockIdx.x * kParseWarps >= total) return;
  for (uint32_t i = threadIdx.x; i < sizeof(SchemaTable) / 4; i += blockDim.x)
    reinterpret_cast<uint32_t*>(&sch)[i] = reinterpret_cast<const uint32_t*>(tab)[i];
  for (uint32_t i = threadIdx.x; i <= n_rings; i += blockDim.x) prefix[i] = ix.rec_prefix[i];
  __syncthreads();
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t gw = blockIdx.x * kParseWarps + warp, nw = gridDim.x * kParseWarps;
  for (uint32_t d = gw; d < total; d += nw) {
    // ring of dense record d: the last r < n_rings with prefix[r] <= d (empty rings share a prefix)
    uint32_t lo = 0, hi = n_rings;
    while (hi - lo > 1) {
      uint32_t mid = (lo + hi) >> 1;
      if (prefix[mid] <= d) lo = mid; else hi = mid;
    }
    parse_record(ix, sch, cfg, d, lo, lo * ix.recs_per_ring + (d - prefix[lo]), heads[warp], lane, total == 1);
    __syncwarp();  // the head buffer is free for the warp's next record
  }
  TL_END(cfg, TL_PARSE);
}

}  // namespace

cudaError_t launch_parse(const IndexDev& ix, const SchemaTable* schemas, const ConfigDev& cfg, uint32_t n_rings,
                         int sms, cudaStream_t s) {
  prof_mark(PROF_PARSE, true, s);
  // no more CTAs than the index's record slots of these rings can occupy
  const uint64_t bound = (uint64_t)ix.recs_per_ring * n_rings;
  const uint64_t want = (bound + kParseWarps - 1) / kParseWarps, most = (uint64_t)sms * CRK_PARSE_CTAS_PER_SM;
  const uint32_t grid = (uint32_t)(want < most ? want : most);
  CRK_LAUNCH(pdl_of(cfg), parse_kernel, grid ? grid : 1, kParseWarps * 32, 0, s, ix, schemas, cfg, n_rings);
  prof_mark(PROF_PARSE, false, s);
  return cudaGetLastError();
}

}  // namespace crk
