// Probe: cost of one hop of a record-marking header chain (p -> p + 4 + len(be32(p))) walked by one warp,
// with the chain in HBM, and the effect of L2 prefetch schemes on it.  Prints JSON (ns per hop).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o chase_probe chase_probe.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include <vector>

__device__ __forceinline__ uint32_t bswap32(uint32_t x) { return __byte_perm(x, 0, 0x0123); }

// mode 0: no prefetch; 1: UBLKPF chunk/lead by lane 0 in the loop; 2: helper warps (1..7) prefetch lines
// (prefetch.global.L2) up to `lead` past the published walk position; 3: helper warps LDG one word per
// line; 4: helper warps UBLKPF chunks
__global__ void chase_kernel(const uint8_t* base, uint64_t n, uint64_t hops, int mode, uint32_t chunk, uint64_t lead,
                             uint64_t* out, int ld) {
  __shared__ volatile uint64_t pos;
  __shared__ volatile int done;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) { pos = 0; done = 0; }
  __syncthreads();
  if (warp == 0) {
    uint64_t q = 0, pf = 0, k = 0;
    const long long t0 = clock64();
    for (; k < hops; ++k) {
      if (q + 8 > n) break;
      if (mode == 1 && lane == 0) {
        const uint64_t want = q + lead < n ? q + lead : n;
        for (int i = 0; i < 4 && pf < want; ++i) {
          uint32_t b = chunk;
          if (pf + b > n) b = (uint32_t)((n - pf) & ~15ull);
          if (b) asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(base + pf), "r"(b) : "memory");
          pf += chunk;
        }
      }
      const uint64_t a = q & ~3ull;
      uint32_t w0, w1;
      if (ld == 0) {
        w0 = __ldg(reinterpret_cast<const uint32_t*>(base + a));
        w1 = __ldg(reinterpret_cast<const uint32_t*>(base + a + 4));
      } else if (ld == 1) {
        w0 = __ldcg(reinterpret_cast<const uint32_t*>(base + a));
        w1 = __ldcg(reinterpret_cast<const uint32_t*>(base + a + 4));
      } else if (ld == 2) {
        w0 = *reinterpret_cast<const uint32_t*>(base + a);
        w1 = *reinterpret_cast<const uint32_t*>(base + a + 4);
      } else if (ld == 3) {
        w0 = __ldcv(reinterpret_cast<const uint32_t*>(base + a));
        w1 = __ldcv(reinterpret_cast<const uint32_t*>(base + a + 4));
      } else {  // one load of the aligned 8 bytes when the header does not straddle it
        const uint64_t a8 = q & ~7ull;
        const uint64_t x = __ldcg(reinterpret_cast<const unsigned long long*>(base + a8));
        if ((q & 7) <= 4) {
          const uint32_t sh = 8 * (uint32_t)(q & 7);
          w0 = (uint32_t)(x >> sh);
          w1 = 0;
          const uint32_t h = bswap32(w0);
          q += 4 + (h & 0x7fffffffu);
          if (mode >= 2 && lane == 0 && (k & 3) == 0) pos = q;
          continue;
        }
        w0 = (uint32_t)(x >> 32);
        w1 = __ldcg(reinterpret_cast<const uint32_t*>(base + a8 + 8));
        const uint32_t sh = 8 * (uint32_t)(q & 3);
        const uint32_t h = bswap32(__funnelshift_r(w0, w1, sh));
        q += 4 + (h & 0x7fffffffu);
        if (mode >= 2 && lane == 0 && (k & 3) == 0) pos = q;
        continue;
      }
      const uint32_t h = bswap32(__funnelshift_r(w0, w1, 8 * (uint32_t)(q & 3)));
      q += 4 + (h & 0x7fffffffu);
      if (mode >= 2 && lane == 0 && (k & 3) == 0) pos = q;
    }
    const long long t1 = clock64();
    if (lane == 0) { out[0] = k; out[1] = (uint64_t)(t1 - t0); out[2] = q; done = 1; }
  } else if (mode >= 2) {
    const uint32_t ht = threadIdx.x - 32, nh = blockDim.x - 32;
    uint64_t pf = 0;
    uint32_t sink = 0;
    while (!done) {
      const uint64_t p = pos;
      uint64_t want = p + lead < n ? p + lead : n;
      if (pf < (p & ~127ull)) pf = p & ~127ull;
      if (mode == 4) {
        // helper warp 1 lane 0 issues bulk prefetches
        if (ht == 0) {
          while (pf < want) {
            uint32_t b = chunk;
            if (pf + b > n) b = (uint32_t)((n - pf) & ~15ull);
            if (b) asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(base + pf), "r"(b) : "memory");
            pf += chunk;
          }
        }
        continue;
      }
      // lines [pf, want): thread ht takes lines pf + 128 * (ht + nh * i)
      for (uint64_t l = pf + 128ull * ht; l < want; l += 128ull * nh) {
        if (mode == 2) asm volatile("prefetch.global.L2 [%0];" ::"l"(base + l));
        else sink += __ldcg(reinterpret_cast<const uint32_t*>(base + l));
      }
      if (want > pf) pf = want;  // every helper thread walks the same schedule
    }
    if (sink == 0x12345678u) out[3] = sink;
  }
}

__global__ void touch_kernel(const uint8_t* base, uint64_t n, uint32_t* sink) {
  uint32_t s = 0;
  for (uint64_t i = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) * 16; i < n; i += 16ull * gridDim.x * blockDim.x)
    s += reinterpret_cast<const uint4*>(base + i)->x;
  if (s == 0x12345678u) *sink = s;
}

int main(int argc, char** argv) {
  const uint64_t n = argc > 1 ? strtoull(argv[1], 0, 0) : (256ull << 20);
  const uint32_t maxlen = argc > 2 ? (uint32_t)strtoul(argv[2], 0, 0) : 65536;
  std::vector<uint8_t> h(n + 64);
  uint64_t s = 0x9E3779B97F4A7C15ull;
  auto rnd = [&]() { s ^= s << 13; s ^= s >> 7; s ^= s << 17; return s; };
  for (uint64_t i = 0; i < n; ++i) h[i] = (uint8_t)rnd();
  uint64_t q = 0, hops = 0;
  while (q + 8 + maxlen < n) {
    const uint32_t len = 1 + (uint32_t)(rnd() % maxlen);
    h[q] = (uint8_t)(len >> 24); h[q + 1] = (uint8_t)(len >> 16); h[q + 2] = (uint8_t)(len >> 8); h[q + 3] = (uint8_t)len;
    q += 4 + len;
    ++hops;
  }
  uint8_t* d;
  uint64_t* o;
  uint32_t* sink;
  cudaMalloc(&d, n + 64);
  cudaMalloc(&o, 64);
  cudaMalloc(&sink, 64);
  cudaMalloc(&sink, 64);
  uint8_t* flush;
  cudaMalloc(&flush, 512ull << 20);
  cudaMemcpy(d, h.data(), n + 64, cudaMemcpyHostToDevice);
  struct V { int mode; uint32_t chunk; uint64_t lead; int warm; const char* name; int ld; };
  V vs[] = {{0, 0, 0, 0, "none", 0}, {0, 0, 0, 1, "warm_nc", 0}, {0, 0, 0, 1, "warm_cg", 1},
            {0, 0, 0, 1, "warm_ca", 2}, {0, 0, 0, 1, "warm_cv", 3}, {0, 0, 0, 1, "warm_cg8", 4},
            {0, 0, 0, 0, "cold_cg", 1}, {0, 0, 0, 0, "cold_cg8", 4},
            {4, 65536, 1 << 20, 0, "helper_ublkpf64k_1m_nc", 0}, {4, 65536, 1 << 20, 0, "helper_ublkpf64k_1m_cg", 1},
            {4, 65536, 1 << 20, 0, "helper_ublkpf64k_1m_cg8", 4}, {4, 131072, 2 << 20, 0, "helper_ublkpf128k_2m_cg8", 4},
            {2, 0, 1 << 20, 0, "helpers_pf_line_1m_cg8", 4}};
  printf("{\"bytes\": %llu, \"maxlen\": %u, \"chain_hops\": %llu", (unsigned long long)n, maxlen,
         (unsigned long long)hops);
  for (const V& v : vs) {
    cudaMemset(flush, 1, 512ull << 20);
    if (v.warm) touch_kernel<<<148 * 4, 256>>>(d, n < (96ull << 20) ? n : (96ull << 20), sink);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    chase_kernel<<<1, 256>>>(d, n, hops, v.mode, v.chunk, v.lead, o, v.ld);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    uint64_t r[3];
    cudaMemcpy(r, o, 24, cudaMemcpyDeviceToHost);
    const uint64_t k = v.warm ? (r[0]) : r[0];
    printf(", \"%s\": {\"hops\": %llu, \"ns_per_hop\": %.1f, \"cycles_per_hop\": %.1f, \"ok\": %d}", v.name,
           (unsigned long long)k, ms * 1e6 / k, (double)r[1] / k, r[2] == q || v.warm);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) { printf(", \"error\": \"%s\"}\n", cudaGetErrorString(e)); return 1; }
  }
  printf("}\n");
  return 0;
}
