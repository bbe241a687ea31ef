// Job builders: turn requests (per-xid decode calls, encode calls) or a whole scanned batch (serve)
// into mover jobs, applying the oracle's semantic checks in its order (oracle/oracle.c
// or_decode_memcpy_h2d, or_decode_item, or_serve).
#include "k_plan.cuh"

namespace crk {

namespace {

// memcpy HtoD requests (oracle or_decode_memcpy_h2d)
__global__ void resolve_h2d_kernel(IndexDev ix, ConfigDev cfg, Scratch sc, uint32_t n, const uint32_t* xids,
                                   void* const* dsts, const uint64_t* dst_bytes, int32_t* statuses, uint64_t* copied,
                                   H2DReq single, uint32_t use_single) {
  pdl_entry();
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const uint32_t xid = use_single ? single.xid : xids[i];
    const uint64_t dst = (uint64_t)(use_single ? single.dst : dsts[i]);
    const uint64_t cap = use_single ? single.dst_bytes : dst_bytes[i];
    int32_t* st_out = use_single ? single.status : statuses + i;
    uint64_t* cp_out = use_single ? single.copied : (copied ? copied + i : nullptr);
    Job job{};
    uint64_t m = 0;
    int st;
    const uint32_t d = xid_lookup(ix, xid);
    if (d == kNotFound) {
      st = CRK_E_XID;
    } else if ((st = ix.p_status[d]) == CRK_OK) {
      if (ix.p_proc[d] != cfg.proc_h2d) {
        st = CRK_E_PROC;
      } else {
        const uint64_t nb = ix.p_count[(uint64_t)d * kMaxItems + 1];
        const uint64_t size = ix.p_value[(uint64_t)d * kMaxItems + 2];
        if (cfg.strict && nb != size) st = CRK_E_SIZE;
        else {
          m = (cfg.strict || nb <= size) ? nb : size;
          if (cap < m) { st = CRK_E_PTR; m = 0; }
          else if (m && !dst) { st = CRK_E_ARG; m = 0; }  // a NULL destination for a non-empty payload
          else job = dec_job(ix, dst, m, ix.p_off[(uint64_t)d * kMaxItems + 1], d, 1);
        }
      }
    }
    if (st != CRK_OK) m = 0;
    sc.jobs[i] = job;
    *st_out = st;
    if (cp_out) *cp_out = m;
    if (use_single) plan_single_job(sc, cfg, job);  // n == 1: no planning launch
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) { sc.counters[1] = n; sc.counters[4] = n; }
}

// typed / opaque argument requests (oracle or_decode_item)
__global__ void resolve_items_kernel(IndexDev ix, ConfigDev cfg, Scratch sc, uint32_t n, const crk_item_req* reqs,
                                     crk_item_req single, uint32_t use_single) {
  pdl_entry();
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const crk_item_req r = use_single ? single : reqs[i];
    Job job{};
    uint64_t cnt = 0;
    int st;
    const uint32_t d = xid_lookup(ix, r.xid);
    if (d == kNotFound) {
      st = CRK_E_XID;
    } else if ((st = ix.p_status[d]) == CRK_OK) {
      const uint64_t b = (uint64_t)d * kMaxItems + r.arg_no;
      const uint32_t es = elem_size_k(r.kind);
      if (r.arg_no >= ix.p_nitems[d] || ix.p_kind[b] != r.kind || es == 0) {
        st = CRK_E_ARG;
      } else if (ix.p_count[b] > r.max_count) {
        st = CRK_E_SIZE;
      } else if ((ix.p_count[b] && !r.dst) || ((uint64_t)r.dst % es) != 0) {
        st = CRK_E_ARG;  // NULL or misaligned destination: the element swap works in element lanes
      } else {
        cnt = ix.p_count[b];
        job = dec_job(ix, (uint64_t)r.dst, cnt * es, ix.p_off[b], d, es);
      }
    }
    sc.jobs[i] = job;
    *r.status = st;
    if (r.count) *r.count = cnt;
    if (use_single) plan_single_job(sc, cfg, job);  // n == 1: no planning launch
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) { sc.counters[1] = n; sc.counters[4] = n; }
}

__global__ void serve_plan1_kernel(IndexDev ix, ConfigDev cfg, Scratch sc, uint64_t region_base,
                                   uint64_t region_bytes) {
  pdl_entry();
  const uint32_t total = *ix.total;
  uint64_t* wire = sc.scan_tmp;  // reply wire sizes -> prefix
  for (uint32_t d = blockIdx.x * blockDim.x + threadIdx.x; d < total; d += gridDim.x * blockDim.x) {
    int st;
    int32_t err;
    uint64_t Ll;
    Job job;
    serve_decide(ix, cfg, d, region_base, region_bytes, st, err, Ll, job, total == 1);
    ix.s_status[d] = st;
    ix.s_reply_err[d] = err;
    const uint64_t w = err >= 0 ? wire_of(Ll, cfg.F) : 0;
    ix.s_reply_wire[d] = w;
    wire[d] = w;
    sc.jobs[d] = job;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) { sc.counters[1] = 2 * total; sc.counters[4] = total; }
  if (!cfg.proc_stripe) return;
  // striped memcpys (reading R22): the last block, once every stripe has decided, gives the leads of complete
  // parents their reply and empties the parent table for the next step
  __shared__ uint32_t last;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    last = atomicAdd(ix.stripe_n + 1, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!last) return;
  __threadfence();
  const uint32_t n = __ldcg(ix.stripe_n);
  for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) {
    const StripeEnt* e = ix.stripe + ix.stripe_list[i];
    const uint32_t d = __ldcg(&e->lead);
    if (d != ~0u && __ldcg(&e->good) != 0 && ~__ldcg(&e->landed_c) == __ldcg(&e->total)) {
      const uint64_t w = wire_of(28, cfg.F);
      ix.s_reply_err[d] = 0;
      ix.s_reply_wire[d] = w;
      wire[d] = w;
    }
  }
  __syncthreads();
  stripe_clear(ix, n, threadIdx.x, blockDim.x);
  __syncthreads();
  if (threadIdx.x == 0) {
    ix.stripe_n[0] = 0;
    ix.stripe_n[1] = 0;
  }
}

// pass 2: reply cursors (prefix of wire sizes within each ring) and the encode jobs
__global__ void serve_plan2_kernel(IndexDev ix, ConfigDev cfg, Scratch sc, SendRingsParam S) {
  pdl_entry();
  const uint32_t total = *ix.total;
  const uint64_t* pre = sc.scan_tmp;
  if (blockIdx.x == 0)
    for (uint32_t r = threadIdx.x; r < S.n_rings; r += blockDim.x) sc.out_rings[r] = S.r[r];
  for (uint32_t d = blockIdx.x * blockDim.x + threadIdx.x; d < total; d += gridDim.x * blockDim.x) {
    const uint32_t ring = ix.p_ring[d];
    const uint32_t first = ix.rec_prefix[ring], end = ix.rec_prefix[ring + 1];
    const uint64_t w = ix.s_reply_wire[d];
    const uint64_t off = (S.doorbell ? S.doorbell[2 * S.n_rings + ring] : S.off[ring]) + (pre[d] - pre[first]);
    const int32_t err = ix.s_reply_err[d];
    ix.s_reply_off[d] = err >= 0 ? off : 0;  // (the oracle's convention: 0 when the record has no reply)
    sc.jobs[total + d] = serve_reply_job(ix, cfg, sc, d, ring, err, off, w);
    if (d + 1 == end) ix.res[ring].reply_bytes = pre[d] + w - pre[first];
  }
}

// Small batches: one block of kSmallServe threads runs plan_small_block (k_plan.cuh).
__global__ void __launch_bounds__(kSmallServe) serve_plan_small_kernel(IndexDev ix, ConfigDev cfg, Scratch sc,
                                                                       SendRingsParam S, uint64_t region_base,
                                                                       uint64_t region_bytes) {
  pdl_entry();
  __shared__ uint64_t warp_sums[32];
  __shared__ uint64_t ring_first_pre[kMaxRings];
  TL_BEGIN(cfg, TL_PLAN);
  plan_small_block(ix, cfg, sc, S, region_base, region_bytes, warp_sums, ring_first_pre);
  TL_END(cfg, TL_PLAN);
}

__global__ void put_enc_jobs_kernel(Scratch sc, ConfigDev cfg, EncJobParam p, RingDesc out) {
  pdl_entry();
  if (threadIdx.x == 0) {
    for (uint32_t j = 0; j < p.n_jobs; ++j) sc.jobs[j] = p.jobs[j];
    sc.out_rings[0] = out;
    sc.counters[1] = p.n_jobs;
    sc.counters[4] = p.n_jobs;
    if (p.n_jobs == 1) plan_single_job(sc, cfg, p.jobs[0]);  // no planning launch
  }
  for (uint32_t i = threadIdx.x; i < p.n_pieces; i += blockDim.x) sc.pieces[i] = p.pieces[i];
}

__global__ void d2h_sizes_kernel(Scratch sc, ConfigDev cfg, uint32_t n, const uint64_t* bytes, const int32_t* errs) {
  pdl_entry();
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int32_t err = errs ? errs[i] : 0;
    const uint64_t nb = err == 0 ? bytes[i] : 0;
    const uint64_t Ll = err == 0 ? 32 + nb + pad4(nb) : 28;
    sc.scan_tmp[i] = wire_of(Ll, cfg.F);
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) { sc.counters[1] = n; sc.counters[4] = n; }
}

__global__ void d2h_jobs_kernel(Scratch sc, ConfigDev cfg, uint32_t n, const uint32_t* xids, const void* const* srcs,
                                const uint64_t* bytes, const int32_t* errs, RingDesc out, uint64_t out_off,
                                uint64_t* wire_offs, uint64_t* total_dev, const uint64_t* total_scan) {
  pdl_entry();
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    sc.out_rings[0] = out;
    if (total_dev) *total_dev = *total_scan;
  }
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int32_t err = errs ? errs[i] : 0;
    const uint64_t nb = err == 0 ? bytes[i] : 0;
    const uint64_t off = out_off + sc.scan_tmp[i];
    Piece* P = sc.pieces + 2ull * i;
    reply_words(P[0], xids[i], err, err == 0, nb);
    uint32_t np = 1;
    uint64_t Ll = P[0].nbytes;
    if (err == 0) {
      Piece q{};
      q.type = PIECE_DATA;
      q.loff = 32;
      q.nbytes = nb;
      q.src = (uint64_t)srcs[i];
      q.esize = 1;
      P[1] = q;
      np = 2;
      Ll = 32 + nb + pad4(nb);
    }
    Job job{};
    job.type = JOB_ENC;
    job.out_start = off;
    job.out_end = off + wire_of(Ll, cfg.F);
    job.loff = Ll;
    job.piece0 = 2 * i;
    job.n_pieces = np;
    job.F = cfg.F;
    job.out_ring = 0;
    sc.jobs[i] = job;
    if (wire_offs) wire_offs[i] = off;
  }
}

// ---- generic replies: REPLY header | int err | [one item]
__device__ __forceinline__ uint32_t esize_of(uint32_t kind) { return elem_size_k(kind); }
__device__ __forceinline__ bool kind_var_k(uint32_t k) {
  return k == CRK_K_OPAQUE_VAR || (k >= CRK_K_I32_VAR && k <= CRK_K_F64_VAR);
}
// A request whose item cannot be encoded (count >= 2^32, null or misaligned src) becomes err = CRK_E_ARG.
__device__ __forceinline__ int32_t reply_err_eff(const crk_reply_req& r) {
  if (r.err != 0 || r.kind < CRK_K_OPAQUE_VAR || r.kind > CRK_K_F64_FIX) return r.err;
  const uint32_t es = esize_of(r.kind);
  if (r.count > 0xffffffffull || (r.count && !r.src) || ((uintptr_t)r.src % es) != 0) return CRK_E_ARG;
  return 0;
}
__device__ __forceinline__ uint64_t reply_item_logical(crk_reply_req r) {
  uint64_t L = 28;  // header (24) + err (4)
  r.err = reply_err_eff(r);
  if (r.err != 0 || r.kind == 0 || r.kind > CRK_K_F64_FIX) return L;  // no item (unknown kinds: none)
  if (r.kind == CRK_K_U32) return L + 4;
  if (r.kind == CRK_K_U64) return L + 8;
  const uint64_t nb = r.count * esize_of(r.kind);
  return L + (kind_var_k(r.kind) ? 4 : 0) + nb + pad4(nb);
}

__global__ void replies_sizes_kernel(Scratch sc, ConfigDev cfg, uint32_t n, const crk_reply_req* reqs) {
  pdl_entry();
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    sc.scan_tmp[i] = wire_of(reply_item_logical(reqs[i]), cfg.F);
  if (blockIdx.x == 0 && threadIdx.x == 0) { sc.counters[1] = n; sc.counters[4] = n; }
}

__global__ void replies_jobs_kernel(Scratch sc, ConfigDev cfg, uint32_t n, const crk_reply_req* reqs, RingDesc out,
                                    uint64_t out_off, uint64_t* wire_offs, uint64_t* total_dev,
                                    const uint64_t* total_scan) {
  pdl_entry();
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    sc.out_rings[0] = out;
    if (total_dev) *total_dev = *total_scan;
  }
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    crk_reply_req r = reqs[i];
    r.err = reply_err_eff(r);
    const uint64_t off = out_off + sc.scan_tmp[i];
    const uint64_t Ll = reply_item_logical(r);
    Piece* P = sc.pieces + 2ull * i;
    Piece w{};
    w.type = PIECE_WORDS;
    w.words[0] = r.xid;  // RFC 5531 §9 REPLY, MSG_ACCEPTED, verf AUTH_NONE, SUCCESS
    w.words[1] = 1;
    w.words[6] = (uint32_t)r.err;
    uint32_t nw = 7, np = 1;
    Piece q{};
    const bool item = r.err == 0 && r.kind != 0 && r.kind <= CRK_K_F64_FIX;
    if (item && r.kind == CRK_K_U32) {
      w.words[nw++] = (uint32_t)r.value;
    } else if (item && r.kind == CRK_K_U64) {  // RFC 4506 §4.5: most significant word first
      w.words[nw++] = (uint32_t)(r.value >> 32);
      q.type = PIECE_WORDS;
      q.loff = 32;
      q.nbytes = 4;
      q.words[0] = (uint32_t)r.value;
      np = 2;
    } else if (item) {
      if (kind_var_k(r.kind)) w.words[nw++] = (uint32_t)r.count;
      q.type = PIECE_DATA;
      q.loff = 4ull * nw;
      q.nbytes = r.count * esize_of(r.kind);
      q.src = (uint64_t)r.src;
      q.esize = esize_of(r.kind);
      np = 2;
    }
    w.nbytes = 4ull * nw;
    P[0] = w;
    if (np == 2) P[1] = q;
    Job job{};
    job.type = JOB_ENC;
    job.out_start = off;
    job.out_end = off + wire_of(Ll, cfg.F);
    job.loff = Ll;
    job.piece0 = 2 * i;
    job.n_pieces = np;
    job.F = cfg.F;
    job.out_ring = 0;
    sc.jobs[i] = job;
    if (wire_offs) wire_offs[i] = off;
  }
}

__global__ void lens_prep_kernel(Scratch sc, const uint32_t* lens32, uint32_t n) {
  pdl_entry();
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    sc.lens_pool[i] = lens32[i];
    sc.lens_pool[sc.max_lens + i] = (uint64_t)lens32[i] + 4;  // -> wire starts after the scan
  }
}

inline uint32_t blocks_for(uint32_t n, uint32_t per = 256, uint32_t cap = 148 * 16) {
  uint32_t b = (n + per - 1) / per;
  return b == 0 ? 1 : (b > cap ? cap : b);
}

}  // namespace

cudaError_t launch_resolve_h2d(const IndexDev& ix, const ConfigDev& cfg, Scratch& sc, uint32_t n, const uint32_t* xids,
                               void* const* dsts, const uint64_t* dst_bytes, int32_t* statuses, uint64_t* copied,
                               const H2DReq* single, cudaStream_t s) {
  H2DReq one{};
  if (single) one = *single;
  CRK_LAUNCH(pdl_of(cfg), resolve_h2d_kernel, blocks_for(n), 256, 0, s, ix, cfg, sc, n, xids, dsts, dst_bytes, statuses, copied, one,
                                                    single ? 1u : 0u);
  return cudaGetLastError();
}

cudaError_t launch_resolve_items(const IndexDev& ix, const ConfigDev& cfg, Scratch& sc, uint32_t n,
                                 const crk_item_req* reqs, const crk_item_req* single, cudaStream_t s) {
  crk_item_req one{};
  if (single) one = *single;
  CRK_LAUNCH(pdl_of(cfg), resolve_items_kernel, blocks_for(n), 256, 0, s, ix, cfg, sc, n, reqs, one, single ? 1u : 0u);
  return cudaGetLastError();
}

cudaError_t launch_serve_plan(const IndexDev& ix, const ConfigDev& cfg, Scratch& sc, uint32_t n_rings,
                              const crk_ring* send_rings, const uint64_t* send_offs, uint64_t region_base,
                              uint64_t region_bytes, const uint64_t* doorbell, cudaStream_t s) {
  const uint32_t bound = ix.max_records;
  prof_mark(PROF_PLAN, true, s);
  CRK_LAUNCH(pdl_of(cfg), serve_plan1_kernel, blocks_for(bound), 256, 0, s, ix, cfg, sc, region_base, region_bytes);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  e = launch_exclusive_scan_u64(sc.scan_tmp, bound, ix.total, nullptr, sc, s);
  if (e != cudaSuccess) return e;
  SendRingsParam S{};
  S.n_rings = n_rings;
  for (uint32_t r = 0; r < n_rings; ++r) {
    S.r[r].base = send_rings[r].base;
    S.r[r].mask = send_rings[r].cap - 1;
    S.r[r].head = S.r[r].tail = 0;
    S.off[r] = send_offs ? send_offs[r] : 0;
  }
  S.doorbell = doorbell;
  CRK_LAUNCH(pdl_of(cfg), serve_plan2_kernel, blocks_for(bound), 256, 0, s, ix, cfg, sc, S);
  prof_mark(PROF_PLAN, false, s);
  return cudaGetLastError();
}

cudaError_t launch_serve_plan_small(const IndexDev& ix, const ConfigDev& cfg, Scratch& sc, uint32_t n_rings,
                                    const crk_ring* send_rings, const uint64_t* send_offs, uint64_t region_base,
                                    uint64_t region_bytes, const uint64_t* doorbell, cudaStream_t s) {
  SendRingsParam S{};
  S.n_rings = n_rings;
  for (uint32_t r = 0; r < n_rings; ++r) {
    S.r[r].base = send_rings[r].base;
    S.r[r].mask = send_rings[r].cap - 1;
    S.off[r] = send_offs ? send_offs[r] : 0;
  }
  S.doorbell = doorbell;
  prof_mark(PROF_PLAN, true, s);
  CRK_LAUNCH(pdl_of(cfg), serve_plan_small_kernel, 1, kSmallServe, 0, s, ix, cfg, sc, S, region_base, region_bytes);
  prof_mark(PROF_PLAN, false, s);
  return cudaGetLastError();
}

cudaError_t launch_put_enc_jobs(Scratch& sc, const ConfigDev& cfg, const EncJobParam& p, const RingDesc& out,
                                cudaStream_t s) {
  CRK_LAUNCH(pdl_of(cfg), put_enc_jobs_kernel, 1, 64, 0, s, sc, cfg, p, out);
  return cudaGetLastError();
}

cudaError_t launch_d2h_batch_jobs(Scratch& sc, const ConfigDev& cfg, uint32_t n, const uint32_t* xids,
                                  const void* const* srcs, const uint64_t* bytes, const int32_t* errs,
                                  const RingDesc& out, uint64_t out_off, uint64_t* wire_offs, uint64_t* total,
                                  cudaStream_t s) {
  CRK_LAUNCH(pdl_of(cfg), d2h_sizes_kernel, blocks_for(n), 256, 0, s, sc, cfg, n, bytes, errs);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  uint64_t* tot = sc.scan_tmp + sc.max_jobs + 1;
  e = launch_exclusive_scan_u64(sc.scan_tmp, n, nullptr, tot, sc, s);
  if (e != cudaSuccess) return e;
  CRK_LAUNCH(pdl_of(cfg), d2h_jobs_kernel, blocks_for(n), 256, 0, s, sc, cfg, n, xids, srcs, bytes, errs, out, out_off, wire_offs, total,
                                                 tot);
  return cudaGetLastError();
}

cudaError_t launch_replies_jobs(Scratch& sc, const ConfigDev& cfg, uint32_t n, const crk_reply_req* reqs,
                                const RingDesc& out, uint64_t out_off, uint64_t* wire_offs, uint64_t* total,
                                cudaStream_t s) {
  CRK_LAUNCH(pdl_of(cfg), replies_sizes_kernel, blocks_for(n), 256, 0, s, sc, cfg, n, reqs);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  uint64_t* tot = sc.scan_tmp + sc.max_jobs + 1;
  e = launch_exclusive_scan_u64(sc.scan_tmp, n, nullptr, tot, sc, s);
  if (e != cudaSuccess) return e;
  CRK_LAUNCH(pdl_of(cfg), replies_jobs_kernel, blocks_for(n), 256, 0, s, sc, cfg, n, reqs, out, out_off, wire_offs, total, tot);
  return cudaGetLastError();
}

cudaError_t launch_put_lens(Scratch& sc, const uint32_t* lens32_dev, uint32_t n, cudaStream_t s) {
  CRK_LAUNCH(sc.pdl != 0, lens_prep_kernel, blocks_for(n), 256, 0, s, sc, lens32_dev, n);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  return launch_exclusive_scan_u64(sc.lens_pool + sc.max_lens, n, nullptr, nullptr, sc, s);
}

}  // namespace crk
