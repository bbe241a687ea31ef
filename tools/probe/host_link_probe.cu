// Host-link and staging-path probe (component P1).
//
// Measures, on one B200, the rooflines every later number is divided by:
//   * copy-engine pinned cudaMemcpyAsync H2D, D2H and bidirectional (two streams at once);
//   * SM zero-copy reads of a UVA-mapped pinned host buffer: LDG.128 and cp.async.bulk (TMA 1-D bulk)
//     into shared memory, each written on to HBM;
//   * SM zero-copy writes (STG.128) from HBM into mapped pinned host memory;
//   * the same two SM copy styles HBM -> HBM, for the device-resident roofline.
// Prints one JSON object. Timing: CUDA events, best and median of R runs after warm-up.
//
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o host_link_probe host_link_probe.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <vector>
#include <algorithm>
#include <string>
#include <atomic>
#include <chrono>
#include <cstring>
#include <thread>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "CUDA %s at %s:%d: %s\n", #x, __FILE__, __LINE__, cudaGetErrorString(e)); exit(1);} } while (0)

__device__ __forceinline__ int4 ld_nc(const int4* p) {
  int4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ void st_na(int4* p, int4 v) {
  asm volatile("st.global.L1::no_allocate.v4.s32 [%0], {%1,%2,%3,%4};"
               :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

template <int U>
__global__ void __launch_bounds__(256) ldg_copy(const int4* __restrict__ src, int4* __restrict__ dst, size_t n16) {
  size_t stride = (size_t)gridDim.x * blockDim.x * U;
  for (size_t base = ((size_t)blockIdx.x * blockDim.x) * U + threadIdx.x; base < n16; base += stride) {
    int4 v[U];
#pragma unroll
    for (int j = 0; j < U; ++j) { size_t i = base + (size_t)j * blockDim.x; if (i < n16) v[j] = ld_nc(src + i); }
#pragma unroll
    for (int j = 0; j < U; ++j) { size_t i = base + (size_t)j * blockDim.x; if (i < n16) st_na(dst + i, v[j]); }
  }
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n"
      "W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra W;\n}\n" :: "r"(smem_u32(bar)), "r"(parity) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               :: "r"(smem_u32(sdst)), "l"(gsrc), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}

// 2-stage cp.async.bulk pipeline: tile t of `tile` bytes -> smem -> STG.128 to dst.
__global__ void __launch_bounds__(256) bulk_copy(const uint8_t* __restrict__ src, uint8_t* __restrict__ dst,
                                                 size_t n, uint32_t tile, int stages) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ __align__(8) uint64_t bar[4];
  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) mbar_init(&bar[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  size_t ntiles = n / tile;
  size_t t0 = blockIdx.x;
  // prologue: fill stages-1 stages
  if (threadIdx.x == 0) {
    for (int s = 0; s < stages - 1; ++s) {
      size_t t = t0 + (size_t)s * gridDim.x;
      if (t < ntiles) { mbar_expect_tx(&bar[s], tile); bulk_g2s(smem + (size_t)s * tile, src + t * tile, tile, &bar[s]); }
    }
  }
  uint32_t phase = 0;
  int k = 0;
  for (size_t t = t0; t < ntiles; t += gridDim.x, ++k) {
    int s = k % stages;
    if (threadIdx.x == 0) {
      int sn = (k + stages - 1) % stages;
      size_t tn = t + (size_t)(stages - 1) * gridDim.x;
      if (tn < ntiles) { mbar_expect_tx(&bar[sn], tile); bulk_g2s(smem + (size_t)sn * tile, src + tn * tile, tile, &bar[sn]); }
    }
    mbar_wait(&bar[s], (k / stages) & 1);
    const int4* s4 = reinterpret_cast<const int4*>(smem + (size_t)s * tile);
    int4* d4 = reinterpret_cast<int4*>(dst + t * tile);
    for (uint32_t i = threadIdx.x; i < tile / 16; i += blockDim.x) st_na(d4 + i, s4[i]);
    __syncthreads();
  }
  (void)phase;
}

struct Stat { double best, med; };
static Stat summarize(std::vector<float>& ms, double bytes) {
  std::sort(ms.begin(), ms.end());
  return {bytes / (ms.front() * 1e-3) / 1e9, bytes / (ms[ms.size() / 2] * 1e-3) / 1e9};
}

template <typename F>
static Stat time_it(F f, double bytes, int warm = 3, int reps = 10) {
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  for (int i = 0; i < warm; ++i) f();
  CK(cudaDeviceSynchronize());
  std::vector<float> ms;
  for (int i = 0; i < reps; ++i) {
    CK(cudaEventRecord(a));
    f();
    CK(cudaEventRecord(b));
    CK(cudaEventSynchronize(b));
    float t; CK(cudaEventElapsedTime(&t, a, b)); ms.push_back(t);
  }
  CK(cudaGetLastError());
  return summarize(ms, bytes);
}

// All-GPUs-at-once mode (the 8-GPU roofline is the CONCURRENTLY measured aggregate, not
// 8x one GPU): one host thread per device, each with its own pinned buffers (allocated by that thread after it
// has bound to its device), a spin barrier before every measurement, copy-engine H2D, D2H and both at once on
// all devices together.  Per device: GB/s from its own CUDA events; aggregate: all bytes / the wall-clock span
// from the barrier to the last device's completion.
static void concurrent(int ngpu, size_t n, int reps) {
  std::atomic<int> arrived{0};
  std::atomic<int> gen{0};
  auto barrier = [&](int parties) {
    const int g = gen.load();
    if (arrived.fetch_add(1) + 1 == parties) { arrived.store(0); gen.fetch_add(1); }
    else while (gen.load() == g) std::this_thread::yield();
  };
  struct Res { double h2d, d2h, bi; };
  std::vector<Res> res(ngpu);
  double wall[3] = {0, 0, 0};
  std::vector<std::thread> th;
  for (int g = 0; g < ngpu; ++g) {
    th.emplace_back([&, g] {
      CK(cudaSetDevice(g));
      uint8_t *h_a, *h_b, *d_a, *d_b;
      CK(cudaHostAlloc(&h_a, n, cudaHostAllocPortable));
      CK(cudaHostAlloc(&h_b, n, cudaHostAllocPortable));
      memset(h_a, 1, n); memset(h_b, 2, n);
      CK(cudaMalloc(&d_a, n)); CK(cudaMalloc(&d_b, n));
      cudaStream_t s1, s2;
      CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking)); CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
      cudaEvent_t a, b, c; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b)); CK(cudaEventCreate(&c));
      for (int test = 0; test < 3; ++test) {
        double best = 0;
        for (int r = 0; r < reps + 1; ++r) {
          CK(cudaDeviceSynchronize());
          barrier(ngpu);
          const auto t0 = std::chrono::steady_clock::now();
          CK(cudaEventRecord(a, s1));
          CK(cudaStreamWaitEvent(s2, a));
          if (test != 1) CK(cudaMemcpyAsync(d_a, h_a, n, cudaMemcpyHostToDevice, s1));
          if (test != 0) CK(cudaMemcpyAsync(h_b, d_b, n, cudaMemcpyDeviceToHost, s2));
          CK(cudaEventRecord(c, s2));
          CK(cudaStreamWaitEvent(s1, c));
          CK(cudaEventRecord(b, s1));
          CK(cudaEventSynchronize(b));
          const double span = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
          float ms; CK(cudaEventElapsedTime(&ms, a, b));
          const double bytes = test == 2 ? 2.0 * n : (double)n;
          if (r > 0) best = std::max(best, bytes / (ms * 1e-3) / 1e9);  // r = 0 is the warm-up
          barrier(ngpu);
          if (g == 0 && r > 0) wall[test] = std::max(wall[test], bytes * ngpu / span / 1e9);
        }
        (test == 0 ? res[g].h2d : test == 1 ? res[g].d2h : res[g].bi) = best;
      }
      cudaFreeHost(h_a); cudaFreeHost(h_b); cudaFree(d_a); cudaFree(d_b);
    });
  }
  for (auto& t : th) t.join();
  printf("{\"mode\": \"all_gpus_concurrent\", \"gpus\": %d, \"bytes\": %zu, \"per_gpu\": [", ngpu, n);
  double sh = 0, sd = 0, sb = 0;
  for (int g = 0; g < ngpu; ++g) {
    printf("%s{\"gpu\": %d, \"ce_h2d_gbs\": %.2f, \"ce_d2h_gbs\": %.2f, \"ce_bidir_gbs\": %.2f}", g ? ", " : "", g,
           res[g].h2d, res[g].d2h, res[g].bi);
    sh += res[g].h2d; sd += res[g].d2h; sb += res[g].bi;
  }
  printf("], \"sum_of_per_gpu\": {\"ce_h2d_gbs\": %.2f, \"ce_d2h_gbs\": %.2f, \"ce_bidir_gbs\": %.2f}, "
         "\"aggregate_wall\": {\"ce_h2d_gbs\": %.2f, \"ce_d2h_gbs\": %.2f, \"ce_bidir_gbs\": %.2f}}\n",
         sh, sd, sb, wall[0], wall[1], wall[2]);
}

int main(int argc, char** argv) {
  if (argc > 1 && std::string(argv[1]) == "--all") {  // host_link_probe --all [ngpu] [bytes]
    int ndev = 0;
    CK(cudaGetDeviceCount(&ndev));
    const int ngpu = argc > 2 ? std::min(ndev, atoi(argv[2])) : ndev;
    const size_t bytes = argc > 3 ? strtoull(argv[3], 0, 0) : (size_t)256 << 20;
    concurrent(std::max(1, ngpu), bytes, 5);
    return 0;
  }
  size_t n = (argc > 1 ? strtoull(argv[1], 0, 0) : (size_t)1 << 30);
  int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  cudaDeviceProp prop; CK(cudaGetDeviceProperties(&prop, 0));
  uint8_t *h_a, *h_b, *d_a, *d_b, *hd_a, *hd_b;
  CK(cudaHostAlloc(&h_a, n, cudaHostAllocMapped | cudaHostAllocPortable));
  CK(cudaHostAlloc(&h_b, n, cudaHostAllocMapped | cudaHostAllocPortable));
  memset(h_a, 1, n); memset(h_b, 2, n);
  CK(cudaHostGetDevicePointer((void**)&hd_a, h_a, 0));
  CK(cudaHostGetDevicePointer((void**)&hd_b, h_b, 0));
  CK(cudaMalloc(&d_a, n)); CK(cudaMalloc(&d_b, n));
  CK(cudaMemset(d_a, 3, n)); CK(cudaMemset(d_b, 4, n));
  cudaStream_t s1, s2; CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking)); CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));

  printf("{\"device\": \"%s\", \"sms\": %d, \"bytes\": %zu, \"uva_same_ptr\": %d,\n", prop.name, sms, n, (int)(hd_a == h_a));
  Stat ce_h2d = time_it([&] { CK(cudaMemcpyAsync(d_a, h_a, n, cudaMemcpyHostToDevice, 0)); }, n);
  Stat ce_d2h = time_it([&] { CK(cudaMemcpyAsync(h_b, d_b, n, cudaMemcpyDeviceToHost, 0)); }, n);
  // bidirectional: two streams joined on the legacy stream with events
  cudaEvent_t ev0, e1, e2; CK(cudaEventCreate(&ev0)); CK(cudaEventCreate(&e1)); CK(cudaEventCreate(&e2));
  Stat ce_bi = time_it([&] {
    CK(cudaEventRecord(ev0, 0)); CK(cudaStreamWaitEvent(s1, ev0)); CK(cudaStreamWaitEvent(s2, ev0));
    CK(cudaMemcpyAsync(d_a, h_a, n, cudaMemcpyHostToDevice, s1));
    CK(cudaMemcpyAsync(h_b, d_b, n, cudaMemcpyDeviceToHost, s2));
    CK(cudaEventRecord(e1, s1)); CK(cudaEventRecord(e2, s2));
    CK(cudaStreamWaitEvent(0, e1)); CK(cudaStreamWaitEvent(0, e2)); }, 2.0 * n);
  printf(" \"ce_h2d_gbs\": [%.2f, %.2f], \"ce_d2h_gbs\": [%.2f, %.2f], \"ce_bidir_gbs\": [%.2f, %.2f],\n",
         ce_h2d.best, ce_h2d.med, ce_d2h.best, ce_d2h.med, ce_bi.best, ce_bi.med);

  size_t n16 = n / 16;
  for (int mult : {1, 2, 4, 8}) {
    int grid = sms * mult;
    Stat zr = time_it([&] { ldg_copy<4><<<grid, 256>>>((const int4*)hd_a, (int4*)d_a, n16); }, n);
    Stat zw = time_it([&] { ldg_copy<4><<<grid, 256>>>((const int4*)d_b, (int4*)hd_b, n16); }, n);
    Stat hb = time_it([&] { ldg_copy<4><<<grid, 256>>>((const int4*)d_a, (int4*)d_b, n16); }, 2.0 * n);
    printf(" \"ldg_grid%dx\": {\"zc_read_gbs\": [%.2f, %.2f], \"zc_write_gbs\": [%.2f, %.2f], \"hbm_copy_rw_gbs\": [%.2f, %.2f]},\n",
           mult, zr.best, zr.med, zw.best, zw.med, hb.best, hb.med);
  }
  for (uint32_t tile : {8192u, 16384u, 32768u}) {
    for (int stages : {2, 3, 4}) {
      size_t smem = (size_t)tile * stages;
      if (smem > 200 * 1024) continue;
      CK(cudaFuncSetAttribute(bulk_copy, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      int per_sm = 0;
      CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, bulk_copy, 256, smem));
      int grid = sms * std::max(1, per_sm);
      Stat zr = time_it([&] { bulk_copy<<<grid, 256, smem>>>(hd_a, d_a, n, tile, stages); }, n);
      Stat hb = time_it([&] { bulk_copy<<<grid, 256, smem>>>(d_a, d_b, n, tile, stages); }, 2.0 * n);
      printf(" \"bulk_t%u_s%d\": {\"ctas_per_sm\": %d, \"zc_read_gbs\": [%.2f, %.2f], \"hbm_copy_rw_gbs\": [%.2f, %.2f]},\n",
             tile, stages, per_sm, zr.best, zr.med, hb.best, hb.med);
    }
  }
  // bidirectional: SM zero-copy reads and writes at once (two kernels on two streams), and a CE
  // H2D copy concurrent with SM zero-copy writes
  {
    size_t half16 = n16 / 2;
    Stat bi_sm = time_it([&] {
      CK(cudaEventRecord(ev0, 0)); CK(cudaStreamWaitEvent(s1, ev0)); CK(cudaStreamWaitEvent(s2, ev0));
      ldg_copy<4><<<sms * 2, 256, 0, s1>>>((const int4*)hd_a, (int4*)d_a, half16);
      ldg_copy<4><<<sms * 2, 256, 0, s2>>>((const int4*)d_b, (int4*)hd_b, half16);
      CK(cudaEventRecord(e1, s1)); CK(cudaEventRecord(e2, s2));
      CK(cudaStreamWaitEvent(0, e1)); CK(cudaStreamWaitEvent(0, e2)); }, (double)n);
    Stat ce_sm = time_it([&] {
      CK(cudaEventRecord(ev0, 0)); CK(cudaStreamWaitEvent(s1, ev0)); CK(cudaStreamWaitEvent(s2, ev0));
      CK(cudaMemcpyAsync(d_a, h_a, n / 2, cudaMemcpyHostToDevice, s1));
      ldg_copy<4><<<sms * 2, 256, 0, s2>>>((const int4*)d_b, (int4*)hd_b, half16);
      CK(cudaEventRecord(e1, s1)); CK(cudaEventRecord(e2, s2));
      CK(cudaStreamWaitEvent(0, e1)); CK(cudaStreamWaitEvent(0, e2)); }, (double)n);
    printf(" \"sm_zc_bidir_gbs\": [%.2f, %.2f], \"ce_h2d_plus_sm_zc_write_gbs\": [%.2f, %.2f],\n", bi_sm.best, bi_sm.med,
           ce_sm.best, ce_sm.med);
  }
  // correctness of the bulk path from sysmem
  CK(cudaMemset(d_a, 0, n));
  for (size_t i = 0; i < n; i += 4093) h_a[i] = (uint8_t)(i * 7);
  CK(cudaFuncSetAttribute(bulk_copy, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536));
  bulk_copy<<<sms, 256, 65536>>>(hd_a, d_a, n, 32768, 2);
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(h_b, d_a, n, cudaMemcpyDeviceToHost));
  printf(" \"bulk_from_sysmem_correct\": %s}\n", memcmp(h_a, h_b, n) == 0 ? "true" : "false");
  return 0;
}
