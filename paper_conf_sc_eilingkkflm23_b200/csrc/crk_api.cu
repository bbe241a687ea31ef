// The C ABI (include/crk.h): argument checks, scratch ownership and launch sequences.  No byte of the
// data path is touched here; every step runs in the kernels of k_scan / k_parse / k_prefix / k_plan /
// k_move.
#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>

#include "crk_internal.h"

using namespace crk;

struct crk_ctx {
  int device;
  int sms;
  int move_ctas;
  crk_config cfg;
  ConfigDev cd;
  SchemaTable host_schemas;
  SchemaTable* d_schemas;
  Scratch sc;
  void* block;
};

struct crk_index {
  crk_ctx* ctx;
  int device;  // kept here so destroy does not depend on the context outliving the index
  IndexDev ix;
  void* block;
  crk_ring_result* host_res;  // pinned
};

namespace crk {
static std::atomic<int> g_launches{0};
void count_launch(int n) { g_launches.fetch_add(n, std::memory_order_relaxed); }

// Stage timing with CUDA events recorded on the launching stream (crk_profile_*).
constexpr uint32_t kProfCap = 2048;
struct ProfState {
  bool on = false, created = false;
  cudaEvent_t ev[PROF_STAGES][2][kProfCap];
  uint32_t n[PROF_STAGES] = {0, 0, 0, 0};
};
static ProfState g_prof;
void prof_mark(int stage, bool begin, cudaStream_t s) {
  if (!g_prof.on) return;
  const uint32_t i = g_prof.n[stage];
  if (i >= kProfCap) return;
  cudaEventRecord(g_prof.ev[stage][begin ? 0 : 1][i], s);
  if (!begin) g_prof.n[stage] = i + 1;
}
}  // namespace crk

static thread_local int g_last_cuda = 0;

namespace {

// Makes `dev` current for the call and discards stale non-sticky errors left in the runtime's
// last-error slot by unrelated calls, so CK(cudaGetLastError()) after a launch reports our launch only.
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) == cudaSuccess && prev != dev) cudaSetDevice(dev);
    else prev = -1;
    (void)cudaGetLastError();
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

inline int cuda_fail(cudaError_t e) {
  g_last_cuda = (int)e;
  return CRK_E_CUDA;
}
#define CK(x)                                  \
  do {                                         \
    cudaError_t e_ = (x);                      \
    if (e_ != cudaSuccess) return cuda_fail(e_); \
  } while (0)

inline bool pow2(uint64_t x) { return x && !(x & (x - 1)); }
inline uint64_t pad4(uint64_t n) { return (4 - (n & 3)) & 3; }
inline uint64_t host_wire(uint64_t Ll, uint32_t F) { return Ll + 4 * (Ll == 0 ? 1 : (Ll + F - 1) / F); }

inline bool ring_ok(const crk_ring& r) {
  return r.base && ((uintptr_t)r.base & 255) == 0 && pow2(r.cap) && r.cap >= 256;
}
inline RingDesc ring_desc(const crk_ring& r, uint64_t head, uint64_t tail) {
  RingDesc d;
  d.base = r.base;
  d.mask = r.cap - 1;
  d.head = head;
  d.tail = tail;
  return d;
}
uint32_t elem_size_host(uint32_t kind) {
  switch (kind) {
    case CRK_K_OPAQUE_VAR: case CRK_K_OPAQUE_FIX: return 1;
    case CRK_K_I32_VAR: case CRK_K_U32_VAR: case CRK_K_F32_VAR:
    case CRK_K_I32_FIX: case CRK_K_U32_FIX: case CRK_K_F32_FIX: return 4;
    case CRK_K_I64_VAR: case CRK_K_U64_VAR: case CRK_K_F64_VAR:
    case CRK_K_I64_FIX: case CRK_K_U64_FIX: case CRK_K_F64_FIX: return 8;
    default: return 0;
  }
}
bool kind_valid(uint32_t k) { return k >= CRK_K_U32 && k <= CRK_K_F64_FIX; }
bool kind_var(uint32_t k) { return k == CRK_K_OPAQUE_VAR || (k >= CRK_K_I32_VAR && k <= CRK_K_F64_VAR); }

void add_builtin(SchemaTable& t, uint32_t proc, std::initializer_list<uint32_t> items) {
  Schema& s = t.s[t.n++];
  memset(&s, 0, sizeof(s));
  s.proc = proc;
  for (uint32_t k : items) s.items[s.n_items++] = k;
}

// Validated scan parameters (host-argument checks of crk_rpc_frame_scan / crk_serve).
int scan_param(crk_index* idx, uint32_t n_rings, const crk_ring* rings, const uint64_t* heads,
               const uint64_t* tails, const uint64_t* doorbell, ScanRingsParam& P) {
  if (!rings || (!doorbell && (!heads || !tails)) || n_rings == 0 || n_rings > (uint32_t)kMaxRings ||
      n_rings > idx->ix.max_rings)
    return CRK_E_ARG;
  memset(&P, 0, sizeof(P));
  P.n_rings = n_rings;
  P.doorbell = doorbell;
  for (uint32_t r = 0; r < n_rings; ++r) {
    if (!ring_ok(rings[r])) return CRK_E_ARG;
    if (doorbell) {
      P.r[r] = ring_desc(rings[r], 0, 0);  // cursors come from the doorbell at execution time
      continue;
    }
    if (tails[r] < heads[r] || tails[r] - heads[r] > rings[r].cap) return CRK_E_ARG;
    P.r[r] = ring_desc(rings[r], heads[r], tails[r]);
  }
  return CRK_OK;
}

// A small index (crk_config.fused_front_max_records) over one ring or a small window: one fused launch.
// A window long enough for the chunked multi-CTA scan (k_mscan.cu) goes to the separate kernels even on one
// ring: the single CTA of the fused front end would walk its whole header chain alone -- unless the index
// holds at most fused_front_max_frags fragments, which bounds that walk (the scan stops at the index's
// capacity): then one launch beats the chunked scan's fixed cost (e.g. one 64 MiB memcpy CALL, 1,025 headers).
bool fused_front(const crk_ctx* c, const crk_index* x, uint32_t n_rings, const uint64_t* heads, const uint64_t* tails,
                 const uint64_t* doorbell) {
  uint64_t window = 0;
  for (uint32_t r = 0; !doorbell && heads && tails && r < n_rings; ++r) window += tails[r] - heads[r];
  const bool capped = (uint64_t)x->ix.frags_per_ring * n_rings <= c->cfg.fused_front_max_frags;
  const bool long_window = window > c->cfg.fused_front_max_window && !capped;
  const bool chunkable = !doorbell && c->cfg.scan_chunking == 0 && long_window;
  return x->ix.max_records <= c->cfg.fused_front_max_records && x->ix.max_records <= front_small_threads() &&
         !chunkable && (n_rings == 1 || (!doorbell && !long_window));
}

int run_scan(crk_ctx* ctx, crk_index* idx, uint32_t n_rings, const crk_ring* rings, const uint64_t* heads,
             const uint64_t* tails, cudaStream_t s, const uint64_t* doorbell = nullptr) {
  ScanRingsParam P;
  const int st = scan_param(idx, n_rings, rings, heads, tails, doorbell, P);
  if (st != CRK_OK) return st;
  if (fused_front(ctx, idx, n_rings, heads, tails, doorbell)) {  // scan + parse in one launch
    CK(launch_front_small(idx->ix, ctx->cd, ctx->sc, ctx->d_schemas, P, n_rings, nullptr, nullptr, 0, 0, doorbell,
                          false, s));
    return CRK_OK;
  }
  CK(cudaMemsetAsync(idx->ix.xid_hash, 0xff, sizeof(unsigned long long) * ((uint64_t)idx->ix.hash_mask + 1), s));
  CK(launch_frame_scan(idx->ix, P, ctx->cd, s));
  CK(launch_parse(idx->ix, ctx->d_schemas, ctx->cd, n_rings, ctx->sms, s));
  return CRK_OK;
}

int move(crk_ctx* ctx, const IndexDev* ix, uint32_t bound, cudaStream_t s, uint64_t out_bytes_bound = 0,
         bool planned = false) {
  CK(launch_plan_and_move(ix, ctx->cd, ctx->sc, bound, out_bytes_bound, ctx->sms, ctx->move_ctas, s, planned));
  return CRK_OK;
}

Piece words_piece(uint64_t loff, const uint32_t* w, uint32_t n) {
  Piece p;
  memset(&p, 0, sizeof(p));
  p.type = PIECE_WORDS;
  p.loff = loff;
  p.nbytes = 4ull * n;
  for (uint32_t i = 0; i < n; ++i) p.words[i] = w[i];
  return p;
}
Piece data_piece(uint64_t loff, const void* src, uint64_t nbytes, uint32_t es) {
  Piece p;
  memset(&p, 0, sizeof(p));
  p.type = PIECE_DATA;
  p.loff = loff;
  p.nbytes = nbytes;
  p.src = (uint64_t)src;
  p.esize = es;
  return p;
}

// REPLY(xid) | int err | [err == 0: T data<> (count, elements)]; one encode job
int encode_reply(crk_ctx* ctx, uint32_t xid, const void* src, uint64_t count, uint32_t es, int32_t err, crk_ring out,
                 uint64_t out_off, uint64_t* wire_bytes, cudaStream_t s) {
  if (!ring_ok(out) || !wire_bytes) return CRK_E_ARG;
  if (err == 0 && (count > 0xffffffffull || (count && !src) || ((uintptr_t)src % es) != 0)) return CRK_E_ARG;
  EncJobParam P;
  memset(&P, 0, sizeof(P));
  const uint32_t w[8] = {xid, 1, 0, 0, 0, 0, (uint32_t)err, (uint32_t)count};
  P.pieces[0] = words_piece(0, w, err == 0 ? 8 : 7);
  uint64_t Ll = P.pieces[0].nbytes;
  P.n_pieces = 1;
  if (err == 0) {
    P.pieces[1] = data_piece(32, src, count * es, es);
    P.n_pieces = 2;
    Ll = 32 + count * es + pad4(count * es);
  }
  const uint64_t wire = host_wire(Ll, ctx->cd.F);
  Job& j = P.jobs[0];
  j.type = JOB_ENC;
  j.out_start = out_off;
  j.out_end = out_off + wire;
  j.loff = Ll;
  j.piece0 = 0;
  j.n_pieces = P.n_pieces;
  j.F = ctx->cd.F;
  j.out_ring = 0;
  P.n_jobs = 1;
  *wire_bytes = wire;
  CK(launch_put_enc_jobs(ctx->sc, ctx->cd, P, ring_desc(out, 0, 0), s));
  return move(ctx, nullptr, 1, s, wire, true);
}

int decode_item_one(crk_ctx* ctx, crk_index* idx, uint32_t xid, uint32_t arg_no, uint32_t kind, void* dst,
                    uint64_t max_count, uint64_t* count_dev, int32_t* status_dev, cudaStream_t s) {
  if (!ctx || !idx || !status_dev) return CRK_E_ARG;
  const uint32_t es = elem_size_host(kind);
  if (!es || (max_count && !dst) || ((uintptr_t)dst % es) != 0) return CRK_E_ARG;
  DeviceGuard g(ctx->device);
  crk_item_req r;
  memset(&r, 0, sizeof(r));
  r.xid = xid;
  r.arg_no = arg_no;
  r.kind = kind;
  r.dst = dst;
  r.max_count = max_count;
  r.count = count_dev;
  r.status = status_dev;
  CK(launch_resolve_items(idx->ix, ctx->cd, ctx->sc, 1, nullptr, &r, s));
  return move(ctx, &idx->ix, 1, s, max_count * es + 1, true);
}

}  // namespace

extern "C" {

void crk_config_init(crk_config* c) {
  if (!c) return;
  memset(c, 0, sizeof(*c));
  c->frag_payload = 65536;
  c->strict = 1;
  c->max_record_bytes = 1ull << 32;
  c->prog = 0x20000099;
  c->vers = 1;
  c->proc_h2d = 1;
  c->proc_d2h = 2;
  c->scan_stride_guess = 0;
  c->tile_bytes = 32768;
  c->max_jobs = 1u << 20;
  c->ctas_per_sm = 0;
  c->scan_threads = 256;
  c->mover_stages = 3;
  c->mover_run = 8;
  c->mover_tail_tiles = 2;
  c->mover_reserve_ctas = 0;
  c->fused_front_max_records = 128;
  c->fused_front_max_window = 1ull << 20;
  c->fused_front_max_frags = 4096;
  c->proc_h2d_stripe = 3;
  c->lean_steps = 1;
  c->lean_backoff = 16;
}

int crk_ctx_create(int device, const crk_config* cfg_in, crk_ctx** out) {
  if (!out) return CRK_E_ARG;
  *out = nullptr;
  crk_config cfg;
  if (cfg_in) cfg = *cfg_in; else crk_config_init(&cfg);
  if (cfg.frag_payload == 0 || cfg.frag_payload > 0x7fffffffu || !pow2(cfg.tile_bytes) || cfg.tile_bytes < 1024 ||
      cfg.tile_bytes > (1u << 20) || cfg.max_jobs == 0 || cfg.proc_h2d == cfg.proc_d2h || cfg.scan_threads < 64 ||
      cfg.scan_threads > 1024 || (cfg.scan_threads & 63) || cfg.mover_stages < 2 || cfg.mover_stages > 8 ||
      cfg.mover_run < 1 || cfg.mover_run > 64 || cfg.mover_tail_tiles > 64 || cfg.scan_chunking > 1 ||
      cfg.lean_steps > 1 ||
      (cfg.proc_h2d_stripe && (cfg.proc_h2d_stripe == cfg.proc_h2d || cfg.proc_h2d_stripe == cfg.proc_d2h)))
    return CRK_E_ARG;
  int ndev = 0;
  CK(cudaGetDeviceCount(&ndev));
  if (device < 0 || device >= ndev) return CRK_E_ARG;
  DeviceGuard g(device);
  CK(cudaSetDevice(device));
  crk_ctx* c = new (std::nothrow) crk_ctx;
  if (!c) return CRK_E_CAPACITY;
  memset(c, 0, sizeof(*c));
  c->device = device;
  c->cfg = cfg;
  CK(cudaDeviceGetAttribute(&c->sms, cudaDevAttrMultiProcessorCount, device));
  int occ = cfg.ctas_per_sm ? (int)cfg.ctas_per_sm : mover_occupancy(cfg.tile_bytes, cfg.mover_stages);
  c->move_ctas = c->sms * (occ > 0 ? occ : 1);
  if (cfg.mover_max_ctas && (uint32_t)c->move_ctas > cfg.mover_max_ctas) c->move_ctas = (int)cfg.mover_max_ctas;
  if (2ull * cfg.mover_reserve_ctas >= (uint64_t)c->move_ctas) { delete c; return CRK_E_ARG; }
  ConfigDev& d = c->cd;
  d.F = cfg.frag_payload;
  d.strict = cfg.strict ? 1 : 0;
  d.prog = cfg.prog;
  d.vers = cfg.vers;
  d.proc_h2d = cfg.proc_h2d;
  d.proc_d2h = cfg.proc_d2h;
  d.guess = cfg.scan_stride_guess ? cfg.scan_stride_guess : cfg.frag_payload;
  d.tile_shift = (uint32_t)__builtin_ctz(cfg.tile_bytes);
  d.max_record_bytes = cfg.max_record_bytes;
  d.scan_threads = cfg.scan_threads;
  d.tl = nullptr;
  d.stages = cfg.mover_stages;
  d.run = cfg.mover_run;
  d.tail = cfg.mover_tail_tiles;
  d.reserve = cfg.mover_reserve_ctas;
  d.no_chunked_scan = cfg.scan_chunking == 1 ? 1u : 0u;
  c->sc.pdl = pdl_of(d) ? 1u : 0u;
  d.proc_stripe = cfg.proc_h2d_stripe;
  d.lean = cfg.lean_steps;
  d.lean_backoff = cfg.lean_backoff;
  add_builtin(c->host_schemas, cfg.proc_h2d, {CRK_K_U64, CRK_K_OPAQUE_VAR, CRK_K_U64});
  add_builtin(c->host_schemas, cfg.proc_d2h, {CRK_K_U64, CRK_K_U64});
  if (cfg.proc_h2d_stripe)  // ptr, mem, size, parent, offset, total (reading R22)
    add_builtin(c->host_schemas, cfg.proc_h2d_stripe,
                {CRK_K_U64, CRK_K_OPAQUE_VAR, CRK_K_U64, CRK_K_U32, CRK_K_U64, CRK_K_U64});
  // scratch: one block
  Scratch& sc = c->sc;
  sc.max_jobs = cfg.max_jobs;
  sc.max_lens = 1u << 20;
  sc.max_pieces = 2 * cfg.max_jobs;
  const uint64_t scan_blocks = ((uint64_t)(sc.max_jobs > sc.max_lens ? sc.max_jobs : sc.max_lens) + 2047) / 2048 + 2;
  const size_t sz[] = {sizeof(Job) * (size_t)sc.max_jobs, sizeof(Piece) * (size_t)sc.max_pieces, 64,
                       sizeof(uint64_t) * 2 * (size_t)sc.max_lens, sizeof(uint32_t) * (size_t)sc.max_lens,
                       sizeof(unsigned long long) * scan_blocks, sizeof(uint64_t) * ((size_t)sc.max_jobs + 2),
                       sizeof(RingDesc) * kMaxRings, sizeof(SchemaTable), sizeof(uint32_t) * (size_t)sc.max_jobs};
  size_t total = 0, off[10];
  for (int i = 0; i < 10; ++i) { off[i] = total; total += (sz[i] + 255) & ~(size_t)255; }
  cudaError_t e = cudaMalloc(&c->block, total);
  if (e != cudaSuccess) { delete c; return cuda_fail(e); }
  char* b = (char*)c->block;
  sc.jobs = (Job*)(b + off[0]);
  sc.pieces = (Piece*)(b + off[1]);
  sc.counters = (uint32_t*)(b + off[2]);
  sc.lens_pool = (uint64_t*)(b + off[3]);
  sc.lens32 = (uint32_t*)(b + off[4]);
  sc.scan_state = (unsigned long long*)(b + off[5]);
  sc.scan_tmp = (uint64_t*)(b + off[6]);
  sc.out_rings = (RingDesc*)(b + off[7]);
  c->d_schemas = (SchemaTable*)(b + off[8]);
  sc.run_job = (uint32_t*)(b + off[9]);
  e = cudaMemset(c->block, 0, total);
  if (e == cudaSuccess) e = cudaMemcpy(c->d_schemas, &c->host_schemas, sizeof(SchemaTable), cudaMemcpyHostToDevice);
  if (e != cudaSuccess) { cudaFree(c->block); delete c; return cuda_fail(e); }
  *out = c;
  return CRK_OK;
}

void crk_ctx_destroy(crk_ctx* c) {
  if (!c) return;
  DeviceGuard g(c->device);
  cudaFree(c->block);
  delete c;
}

int crk_proc_schema_register(crk_ctx* c, uint32_t proc, const uint32_t* items, uint32_t n) {
  if (!c || (n && !items) || n > (uint32_t)kMaxItems) return CRK_E_ARG;
  if (proc == c->cfg.proc_h2d || proc == c->cfg.proc_d2h || (c->cfg.proc_h2d_stripe && proc == c->cfg.proc_h2d_stripe))
    return CRK_E_ARG;
  for (uint32_t i = 0; i < n; ++i) {
    const uint32_t k = items[i] & 0xff, fixed = items[i] >> 8;
    if (!kind_valid(k) || (kind_var(k) && fixed) || ((k == CRK_K_U32 || k == CRK_K_U64) && fixed)) return CRK_E_ARG;
  }
  SchemaTable& t = c->host_schemas;
  Schema* s = nullptr;
  for (uint32_t i = 0; i < t.n; ++i)
    if (t.s[i].proc == proc) s = &t.s[i];
  if (!s) {
    if (t.n >= (uint32_t)kMaxProcs) return CRK_E_CAPACITY;
    s = &t.s[t.n++];
  }
  memset(s, 0, sizeof(*s));
  s->proc = proc;
  s->n_items = n;
  for (uint32_t i = 0; i < n; ++i) s->items[i] = items[i];
  DeviceGuard g(c->device);
  CK(cudaMemcpy(c->d_schemas, &t, sizeof(SchemaTable), cudaMemcpyHostToDevice));
  return CRK_OK;
}

int crk_index_create(crk_ctx* c, uint32_t max_rings, uint32_t max_frags, uint32_t max_records, crk_index** out) {
  if (!c || !out || max_rings == 0 || max_rings > (uint32_t)kMaxRings || max_frags < max_rings ||
      max_records < max_rings || max_records > (1u << 28))
    return CRK_E_ARG;
  *out = nullptr;
  DeviceGuard g(c->device);
  crk_index* x = new (std::nothrow) crk_index;
  if (!x) return CRK_E_CAPACITY;
  memset(x, 0, sizeof(*x));
  x->ctx = c;
  x->device = c->device;
  IndexDev& ix = x->ix;
  ix.max_rings = max_rings;
  ix.frags_per_ring = max_frags / max_rings;
  ix.recs_per_ring = max_records / max_rings;
  const uint32_t F = ix.frags_per_ring * max_rings, R = ix.recs_per_ring * max_rings;
  ix.max_records = R;
  uint64_t hs = 1;
  while (hs < 2ull * R) hs <<= 1;
  ix.hash_mask = (uint32_t)(hs - 1);
  const uint64_t MI = (uint64_t)R * kMaxItems;
  // chunked-scan scratch (k_mscan.cu): enough chunks for the index's fragment capacity at ~16 fragments per
  // chunk, 64 .. 2048
  const uint32_t CC = std::min<uint32_t>(2048u, std::max<uint32_t>(64u, F / 16));
  ix.ms.chunk_cap = CC;
  const size_t sz[] = {
      sizeof(RingDesc) * max_rings, sizeof(crk_ring_result) * max_rings, sizeof(uint32_t) * (max_rings + 1), 4, 4,
      8 * (size_t)F, 8 * (size_t)F, 4 * (size_t)F,                              // frags
      8 * (size_t)R, 8 * (size_t)R, 4 * (size_t)R, 4 * (size_t)R,               // records
      4 * (size_t)R, 4 * (size_t)R, 4 * (size_t)R, 4 * (size_t)R, 4 * (size_t)R, 4 * (size_t)R,  // parsed scalars
      4 * (size_t)R, 4 * (size_t)R, 4 * (size_t)R,                              // parsed fragment coordinates
      4 * MI, 8 * MI, 8 * MI, 8 * MI,                                           // items
      4 * (size_t)R, 4 * (size_t)R, 8 * (size_t)R, 8 * (size_t)R,               // serve
      8 * (size_t)hs,
      sizeof(uint2) * (size_t)CC * kCand * kLogCap, sizeof(ChainSum) * (size_t)CC * kCand,  // chunked scan
      sizeof(ChunkState) * (size_t)CC, sizeof(ChunkStop) * (size_t)CC, sizeof(RingPlan) * max_rings, 16,
      sizeof(StripeEnt) * (size_t)hs, 4 * (size_t)R, 8};  // striped memcpys
  constexpr int N = sizeof(sz) / sizeof(sz[0]);
  size_t total = 0, off[N];
  for (int i = 0; i < N; ++i) { off[i] = total; total += (sz[i] + 255) & ~(size_t)255; }
  cudaError_t e = cudaMalloc(&x->block, total);
  if (e != cudaSuccess) { delete x; return cuda_fail(e); }
  char* b = (char*)x->block;
  int i = 0;
  ix.rings = (RingDesc*)(b + off[i++]);
  ix.res = (crk_ring_result*)(b + off[i++]);
  ix.rec_prefix = (uint32_t*)(b + off[i++]);
  ix.total = (uint32_t*)(b + off[i++]);
  ix.ticket = (uint32_t*)(b + off[i++]);
  ix.frag_phys = (uint64_t*)(b + off[i++]);
  ix.frag_lstart = (uint64_t*)(b + off[i++]);
  ix.frag_hdr = (uint32_t*)(b + off[i++]);
  ix.rec_begin = (uint64_t*)(b + off[i++]);
  ix.rec_len = (uint64_t*)(b + off[i++]);
  ix.rec_frag0 = (uint32_t*)(b + off[i++]);
  ix.rec_nfrags = (uint32_t*)(b + off[i++]);
  ix.p_slot = (uint32_t*)(b + off[i++]);
  ix.p_ring = (uint32_t*)(b + off[i++]);
  ix.p_xid = (uint32_t*)(b + off[i++]);
  ix.p_proc = (uint32_t*)(b + off[i++]);
  ix.p_status = (int32_t*)(b + off[i++]);
  ix.p_nitems = (uint32_t*)(b + off[i++]);
  ix.p_frag0 = (uint32_t*)(b + off[i++]);
  ix.p_nfrags = (uint32_t*)(b + off[i++]);
  ix.p_flen0 = (uint32_t*)(b + off[i++]);
  ix.p_kind = (uint32_t*)(b + off[i++]);
  ix.p_off = (uint64_t*)(b + off[i++]);
  ix.p_count = (uint64_t*)(b + off[i++]);
  ix.p_value = (uint64_t*)(b + off[i++]);
  ix.s_status = (int32_t*)(b + off[i++]);
  ix.s_reply_err = (int32_t*)(b + off[i++]);
  ix.s_reply_off = (uint64_t*)(b + off[i++]);
  ix.s_reply_wire = (uint64_t*)(b + off[i++]);
  ix.xid_hash = (unsigned long long*)(b + off[i++]);
  ix.ms.log = (uint2*)(b + off[i++]);
  ix.ms.sums = (ChainSum*)(b + off[i++]);
  ix.ms.state = (ChunkState*)(b + off[i++]);
  ix.ms.stops = (ChunkStop*)(b + off[i++]);
  ix.ms.plan = (RingPlan*)(b + off[i++]);
  ix.ms.stats = (uint32_t*)(b + off[i++]);
  ix.stripe = (StripeEnt*)(b + off[i++]);
  ix.stripe_list = (uint32_t*)(b + off[i++]);
  ix.stripe_n = (uint32_t*)(b + off[i++]);
  e = cudaMemset(x->block, 0, total);
  if (e == cudaSuccess) e = cudaMemset(ix.xid_hash, 0xff, 8 * (size_t)hs);
  if (e == cudaSuccess) e = cudaMemset(ix.stripe, 0xff, sizeof(StripeEnt) * (size_t)hs);
  for (uint32_t r = 0; e == cudaSuccess && r < max_rings; ++r)  // no stop recorded
    e = cudaMemset(&ix.ms.plan[r].stop_key, 0xff, sizeof(unsigned long long));
  if (e == cudaSuccess) e = cudaMallocHost(&x->host_res, sizeof(crk_ring_result) * max_rings);
  if (e != cudaSuccess) { cudaFree(x->block); delete x; return cuda_fail(e); }
  *out = x;
  return CRK_OK;
}

void crk_index_destroy(crk_index* x) {
  if (!x) return;
  DeviceGuard g(x->device);
  cudaFree(x->block);
  cudaFreeHost(x->host_res);
  delete x;
}

int crk_index_get_view(const crk_index* x, crk_index_view* v) {
  if (!x || !v) return CRK_E_ARG;
  const IndexDev& ix = x->ix;
  v->max_rings = ix.max_rings;
  v->frags_per_ring = ix.frags_per_ring;
  v->recs_per_ring = ix.recs_per_ring;
  v->max_records = ix.max_records;
  v->frag_phys = ix.frag_phys;
  v->frag_lstart = ix.frag_lstart;
  v->frag_hdr = ix.frag_hdr;
  v->rec_begin = ix.rec_begin;
  v->rec_len = ix.rec_len;
  v->rec_frag0 = ix.rec_frag0;
  v->rec_nfrags = ix.rec_nfrags;
  v->p_slot = ix.p_slot;
  v->p_ring = ix.p_ring;
  v->p_xid = ix.p_xid;
  v->p_proc = ix.p_proc;
  v->p_status = ix.p_status;
  v->p_nitems = ix.p_nitems;
  v->p_kind = ix.p_kind;
  v->p_off = ix.p_off;
  v->p_count = ix.p_count;
  v->p_value = ix.p_value;
  v->serve_status = ix.s_status;
  v->serve_reply_err = ix.s_reply_err;
  v->serve_reply_off = ix.s_reply_off;
  v->serve_reply_wire = ix.s_reply_wire;
  v->ring_results = ix.res;
  v->total_records = ix.total;
  return CRK_OK;
}

int crk_index_ring_results(crk_index* x, uint32_t n_rings, crk_ring_result* host_out, crk_stream_t stream) {
  if (!x || !host_out || n_rings > x->ix.max_rings) return CRK_E_ARG;
  DeviceGuard g(x->ctx->device);
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaMemcpyAsync(x->host_res, x->ix.res, sizeof(crk_ring_result) * n_rings, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  memcpy(host_out, x->host_res, sizeof(crk_ring_result) * n_rings);
  return CRK_OK;
}

int crk_index_ring_results_async(crk_index* x, uint32_t n_rings, crk_ring_result* pinned_out, crk_stream_t stream) {
  if (!x || !pinned_out || n_rings > x->ix.max_rings) return CRK_E_ARG;
  DeviceGuard g(x->ctx->device);
  CK(cudaMemcpyAsync(pinned_out, x->ix.res, sizeof(crk_ring_result) * n_rings, cudaMemcpyDeviceToHost,
                     (cudaStream_t)stream));
  return CRK_OK;
}

int crk_ring_copy(crk_ring dst, crk_ring src, uint64_t head, uint64_t tail, crk_stream_t stream) {
  if (!ring_ok(dst) || !ring_ok(src) || tail < head || tail - head > dst.cap || tail - head > src.cap)
    return CRK_E_ARG;
  for (uint64_t c = head; c < tail;) {  // contiguous pieces: neither side wraps inside a piece
    const uint64_t os = c & (src.cap - 1), od = c & (dst.cap - 1);
    uint64_t n = tail - c;
    if (n > src.cap - os) n = src.cap - os;
    if (n > dst.cap - od) n = dst.cap - od;
    CK(cudaMemcpyAsync(dst.base + od, src.base + os, n, cudaMemcpyDefault, (cudaStream_t)stream));
    c += n;
  }
  return CRK_OK;
}

int crk_rpc_frame_scan(crk_ctx* c, crk_index* x, uint32_t n_rings, const crk_ring* rings, const uint64_t* heads,
                       const uint64_t* tails, crk_stream_t stream) {
  if (!c || !x || x->ctx != c) return CRK_E_ARG;
  DeviceGuard g(c->device);
  return run_scan(c, x, n_rings, rings, heads, tails, (cudaStream_t)stream);
}

int crk_xdr_decode_memcpy_h2d(crk_ctx* c, crk_index* x, uint32_t xid, void* dst, uint64_t dst_bytes,
                              int32_t* status_dev, uint64_t* copied_dev, crk_stream_t stream) {
  if (!c || !x || !status_dev || (dst_bytes && !dst)) return CRK_E_ARG;
  DeviceGuard g(c->device);
  H2DReq r;
  r.xid = xid;
  r.dst = dst;
  r.dst_bytes = dst_bytes;
  r.status = status_dev;
  r.copied = copied_dev;
  cudaStream_t s = (cudaStream_t)stream;
  CK(launch_resolve_h2d(x->ix, c->cd, c->sc, 1, nullptr, nullptr, nullptr, nullptr, nullptr, &r, s));
  return move(c, &x->ix, 1, s, dst_bytes + 1, true);
}

int crk_xdr_decode_memcpy_h2d_batch(crk_ctx* c, crk_index* x, uint32_t n, const uint32_t* xids, void* const* dsts,
                                    const uint64_t* dst_bytes, int32_t* statuses, uint64_t* copied,
                                    crk_stream_t stream) {
  if (!c || !x || n > c->sc.max_jobs || (n && (!xids || !dsts || !dst_bytes || !statuses))) return CRK_E_ARG;
  if (n == 0) return CRK_OK;
  DeviceGuard g(c->device);
  cudaStream_t s = (cudaStream_t)stream;
  CK(launch_resolve_h2d(x->ix, c->cd, c->sc, n, xids, dsts, dst_bytes, statuses, copied, nullptr, s));
  return move(c, &x->ix, n, s);
}

#define CRK_DEC_ARRAY(name, T, K)                                                                              \
  int crk_xdr_decode_array_##name(crk_ctx* c, crk_index* x, uint32_t xid, uint32_t arg_no, T* dst,              \
                                  uint64_t max_count, uint64_t* count_dev, int32_t* status_dev,                \
                                  crk_stream_t stream) {                                                       \
    return decode_item_one(c, x, xid, arg_no, K, dst, max_count, count_dev, status_dev, (cudaStream_t)stream); \
  }
CRK_DEC_ARRAY(i32, int32_t, CRK_K_I32_VAR)
CRK_DEC_ARRAY(u32, uint32_t, CRK_K_U32_VAR)
CRK_DEC_ARRAY(i64, int64_t, CRK_K_I64_VAR)
CRK_DEC_ARRAY(u64, uint64_t, CRK_K_U64_VAR)
CRK_DEC_ARRAY(f32, float, CRK_K_F32_VAR)
CRK_DEC_ARRAY(f64, double, CRK_K_F64_VAR)
#undef CRK_DEC_ARRAY

int crk_xdr_decode_opaque(crk_ctx* c, crk_index* x, uint32_t xid, uint32_t arg_no, void* dst, uint64_t max_count,
                          uint64_t* count_dev, int32_t* status_dev, crk_stream_t stream) {
  return decode_item_one(c, x, xid, arg_no, CRK_K_OPAQUE_VAR, dst, max_count, count_dev, status_dev,
                         (cudaStream_t)stream);
}

int crk_xdr_decode_items_batch(crk_ctx* c, crk_index* x, uint32_t n, const crk_item_req* reqs, crk_stream_t stream) {
  if (!c || !x || n > c->sc.max_jobs || (n && !reqs)) return CRK_E_ARG;
  if (n == 0) return CRK_OK;
  DeviceGuard g(c->device);
  cudaStream_t s = (cudaStream_t)stream;
  CK(launch_resolve_items(x->ix, c->cd, c->sc, n, reqs, nullptr, s));
  return move(c, &x->ix, n, s);
}

uint64_t crk_wire_size_d2h(uint64_t bytes, int32_t cuda_err, uint32_t F) {
  if (F == 0) return 0;
  const uint64_t Ll = cuda_err == 0 ? 32 + bytes + pad4(bytes) : 28;
  return host_wire(Ll, F);
}

int crk_xdr_encode_memcpy_d2h(crk_ctx* c, uint32_t xid, const void* src, uint64_t bytes, int32_t cuda_err,
                              crk_ring out, uint64_t out_off, uint64_t* wire_bytes, crk_stream_t stream) {
  if (!c) return CRK_E_ARG;
  DeviceGuard g(c->device);
  return encode_reply(c, xid, src, bytes, 1, cuda_err, out, out_off, wire_bytes, (cudaStream_t)stream);
}

int crk_xdr_encode_memcpy_d2h_batch(crk_ctx* c, uint32_t n, const uint32_t* xids, const void* const* srcs,
                                    const uint64_t* bytes, const int32_t* cuda_errs, crk_ring out, uint64_t out_off,
                                    uint64_t* wire_offs, uint64_t* total_dev, crk_stream_t stream) {
  if (!c || n > c->sc.max_jobs || !ring_ok(out) || (n && (!xids || !srcs || !bytes))) return CRK_E_ARG;
  if (n == 0) return CRK_OK;
  DeviceGuard g(c->device);
  cudaStream_t s = (cudaStream_t)stream;
  CK(launch_d2h_batch_jobs(c->sc, c->cd, n, xids, srcs, bytes, cuda_errs, ring_desc(out, 0, 0), out_off, wire_offs,
                           total_dev, s));
  return move(c, nullptr, n, s);
}

int crk_rpc_encode_replies_batch(crk_ctx* c, uint32_t n, const crk_reply_req* reqs, crk_ring out, uint64_t out_off,
                                 uint64_t* wire_offs, uint64_t* total_dev, crk_stream_t stream) {
  if (!c || n > c->sc.max_jobs || !ring_ok(out) || (n && !reqs)) return CRK_E_ARG;
  if (n == 0) return CRK_OK;
  DeviceGuard g(c->device);
  cudaStream_t s = (cudaStream_t)stream;
  CK(launch_replies_jobs(c->sc, c->cd, n, reqs, ring_desc(out, 0, 0), out_off, wire_offs, total_dev, s));
  return move(c, nullptr, n, s);
}

#define CRK_ENC_ARRAY(name, T)                                                                                   \
  int crk_xdr_encode_array_##name(crk_ctx* c, uint32_t xid, const T* src, uint64_t count, int32_t err,          \
                                  crk_ring out, uint64_t out_off, uint64_t* wire_bytes, crk_stream_t stream) {  \
    if (!c) return CRK_E_ARG;                                                                                    \
    DeviceGuard g(c->device);                                                                                    \
    return encode_reply(c, xid, src, count, sizeof(T), err, out, out_off, wire_bytes, (cudaStream_t)stream);     \
  }
CRK_ENC_ARRAY(i32, int32_t)
CRK_ENC_ARRAY(u32, uint32_t)
CRK_ENC_ARRAY(i64, int64_t)
CRK_ENC_ARRAY(u64, uint64_t)
CRK_ENC_ARRAY(f32, float)
CRK_ENC_ARRAY(f64, double)
#undef CRK_ENC_ARRAY

uint64_t crk_call_logical_size(const crk_item_src* items, uint32_t n) {
  uint64_t L = 40;  // CALL header with AUTH_NONE cred and verf (RFC 5531 §9, §8.2)
  for (uint32_t i = 0; i < n; ++i) {
    const uint32_t k = items[i].kind & 0xff, es = elem_size_host(k);
    if (k == CRK_K_U32) L += 4;
    else if (k == CRK_K_U64) L += 8;
    else L += (kind_var(k) ? 4 : 0) + items[i].count * es + pad4(items[i].count * es);
  }
  return L;
}

int crk_rpc_encode_call(crk_ctx* c, uint32_t xid, uint32_t proc, const crk_item_src* items, uint32_t n_items,
                        const uint32_t* frag_lens, uint32_t n_lens, crk_ring out, uint64_t out_off,
                        uint64_t* wire_bytes, crk_stream_t stream) {
  if (!c || !ring_ok(out) || !wire_bytes || n_items > (uint32_t)kMaxItems || (n_items && !items)) return CRK_E_ARG;
  if (frag_lens && (n_lens == 0 || n_lens > c->sc.max_lens)) return CRK_E_ARG;
  EncJobParam P;
  memset(&P, 0, sizeof(P));
  const uint32_t hdr[10] = {xid, 0, 2, c->cd.prog, c->cd.vers, proc, 0, 0, 0, 0};
  uint64_t L = 0;
  uint32_t np = 0;
  P.pieces[np++] = words_piece(L, hdr, 8);
  L += 32;
  P.pieces[np++] = words_piece(L, hdr + 8, 2);
  L += 8;
  for (uint32_t i = 0; i < n_items; ++i) {
    const crk_item_src& it = items[i];
    const uint32_t k = it.kind & 0xff, es = elem_size_host(k);
    if (!kind_valid(k)) return CRK_E_ARG;
    if (k == CRK_K_U32) {
      const uint32_t w = (uint32_t)it.value;
      P.pieces[np++] = words_piece(L, &w, 1);
      L += 4;
    } else if (k == CRK_K_U64) {
      const uint32_t w[2] = {(uint32_t)(it.value >> 32), (uint32_t)it.value};  // RFC 4506 §4.5
      P.pieces[np++] = words_piece(L, w, 2);
      L += 8;
    } else {
      if (it.count > 0xffffffffull || (it.count && !it.src) || ((uintptr_t)it.src % es) != 0) return CRK_E_ARG;
      if (kind_var(k)) {
        const uint32_t w = (uint32_t)it.count;
        P.pieces[np++] = words_piece(L, &w, 1);
        L += 4;
      }
      P.pieces[np++] = data_piece(L, it.src, it.count * es, es);
      L += it.count * es + pad4(it.count * es);
    }
  }
  P.n_pieces = np;
  Job& j = P.jobs[0];
  j.type = JOB_ENC;
  j.loff = L;
  j.piece0 = 0;
  j.n_pieces = np;
  j.out_start = out_off;
  j.out_ring = 0;
  uint64_t wire;
  DeviceGuard g(c->device);
  cudaStream_t s = (cudaStream_t)stream;
  if (frag_lens) {
    uint64_t sum = 0;
    for (uint32_t i = 0; i < n_lens; ++i) {
      if (frag_lens[i] > 0x7fffffffu) return CRK_E_ARG;
      sum += frag_lens[i];
    }
    if (sum != L) return CRK_E_ARG;
    wire = L + 4ull * n_lens;
    j.F = 0;
    j.lens0 = 0;
    j.n_lens = n_lens;
    CK(cudaMemcpyAsync(c->sc.lens32, frag_lens, sizeof(uint32_t) * n_lens, cudaMemcpyHostToDevice, s));
    CK(launch_put_lens(c->sc, c->sc.lens32, n_lens, s));
  } else {
    wire = host_wire(L, c->cd.F);
    j.F = c->cd.F;
  }
  j.out_end = out_off + wire;
  P.n_jobs = 1;
  *wire_bytes = wire;
  CK(launch_put_enc_jobs(c->sc, c->cd, P, ring_desc(out, 0, 0), s));
  return move(c, nullptr, 1, s, wire, true);
}

}  // extern "C"

namespace {
int run_serve(crk_ctx* c, crk_index* x, uint32_t n_rings, const crk_ring* rings, const uint64_t* heads,
              const uint64_t* tails, const crk_ring* send_rings, const uint64_t* send_offs, uint64_t region_base,
              uint64_t region_bytes, const uint64_t* doorbell, cudaStream_t s) {
  if (!c || !x || x->ctx != c || !send_rings || (!send_offs && !doorbell)) return CRK_E_ARG;
  if (2ull * x->ix.max_records > c->sc.max_jobs) return CRK_E_CAPACITY;
  for (uint32_t r = 0; r < n_rings && r < (uint32_t)kMaxRings; ++r)
    if (!ring_ok(send_rings[r])) return CRK_E_ARG;
  // small step (an index of at most cfg.fused_front_max_records records; one ring, or at most
  // cfg.fused_front_max_window bytes of windows): scan, parse and planning fused into one single-CTA
  // launch, then the mover
  if (fused_front(c, x, n_rings, heads, tails, doorbell)) {
    ScanRingsParam P;
    const int st = scan_param(x, n_rings, rings, heads, tails, doorbell, P);
    if (st != CRK_OK) return st;
    CK(launch_front_small(x->ix, c->cd, c->sc, c->d_schemas, P, n_rings, send_rings, send_offs, region_base,
                          region_bytes, doorbell, true, s));
    CK(launch_mover(&x->ix, c->cd, c->sc, c->cd.run, c->move_ctas, s));
    return CRK_OK;
  }
  int st = run_scan(c, x, n_rings, rings, heads, tails, s, doorbell);
  if (st != CRK_OK) return st;
  if (x->ix.max_records <= kSmallServe) {  // small batch: one planning launch, then the mover
    CK(launch_serve_plan_small(x->ix, c->cd, c->sc, n_rings, send_rings, send_offs, region_base, region_bytes,
                               doorbell, s));
    CK(launch_mover(&x->ix, c->cd, c->sc, c->cd.run, c->move_ctas, s));
    return CRK_OK;
  }
  CK(launch_serve_plan(x->ix, c->cd, c->sc, n_rings, send_rings, send_offs, region_base, region_bytes, doorbell,
                       s));
  return move(c, &x->ix, 2 * x->ix.max_records, s);
}
}  // namespace

struct crk_graph {
  crk_ctx* ctx;
  int device;
  cudaGraph_t graph;
  cudaGraphExec_t exec;
  int launches;  // kernels per replay
};

extern "C" {

int crk_serve(crk_ctx* c, crk_index* x, uint32_t n_rings, const crk_ring* rings, const uint64_t* heads,
              const uint64_t* tails, const crk_ring* send_rings, const uint64_t* send_offs, uint64_t region_base,
              uint64_t region_bytes, crk_stream_t stream) {
  if (!c) return CRK_E_ARG;
  DeviceGuard g(c->device);
  return run_serve(c, x, n_rings, rings, heads, tails, send_rings, send_offs, region_base, region_bytes, nullptr,
                   (cudaStream_t)stream);
}

int crk_serve_graph_create(crk_ctx* c, crk_index* x, uint32_t n_rings, const crk_ring* rings,
                           const crk_ring* send_rings, uint64_t region_base, uint64_t region_bytes,
                           const uint64_t* doorbell, crk_graph** out) {
  if (!c || !x || !doorbell || !out) return CRK_E_ARG;
  *out = nullptr;
  DeviceGuard g(c->device);
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  const bool prof = g_prof.on;
  g_prof.on = false;  // no event nodes inside the graph
  const int l0 = crk::g_launches.load();
  cudaError_t e = cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal);
  int st = CRK_OK;
  if (e == cudaSuccess)
    st = run_serve(c, x, n_rings, rings, nullptr, nullptr, send_rings, nullptr, region_base, region_bytes, doorbell, s);
  cudaGraph_t graph = nullptr;
  const cudaError_t e2 = cudaStreamEndCapture(s, &graph);
  g_prof.on = prof;
  const int nk = crk::g_launches.load() - l0;
  crk::g_launches.fetch_sub(nk);  // launches are counted when the graph is replayed
  cudaStreamDestroy(s);
  if (e != cudaSuccess) return cuda_fail(e);
  if (st != CRK_OK) { if (graph) cudaGraphDestroy(graph); return st; }
  if (e2 != cudaSuccess) return cuda_fail(e2);
  cudaGraphExec_t exec;
  e = cudaGraphInstantiate(&exec, graph, 0);
  if (e != cudaSuccess) { cudaGraphDestroy(graph); return cuda_fail(e); }
  crk_graph* G = new (std::nothrow) crk_graph;
  if (!G) { cudaGraphExecDestroy(exec); cudaGraphDestroy(graph); return CRK_E_CAPACITY; }
  G->ctx = c;
  G->device = c->device;
  G->graph = graph;
  G->exec = exec;
  G->launches = nk;
  *out = G;
  return CRK_OK;
}

int crk_graph_launch(crk_graph* G, crk_stream_t stream) {
  if (!G) return CRK_E_ARG;
  DeviceGuard g(G->device);
  CK(cudaGraphLaunch(G->exec, (cudaStream_t)stream));
  crk::count_launch(G->launches);
  return CRK_OK;
}

void crk_graph_destroy(crk_graph* G) {
  if (!G) return;
  DeviceGuard g(G->device);
  cudaGraphExecDestroy(G->exec);
  cudaGraphDestroy(G->graph);
  delete G;
}

// Diagnostic (not in the public header): the chunked scan's totals for this index (rings resolved by the
// chunked scan, rings that fell back to the one-CTA scan) after synchronising the device.
extern "C" int crk_debug_index_stats(crk_index* x, uint32_t* host4) {
  if (!x || !host4) return CRK_E_ARG;
  DeviceGuard g(x->device);
  if (cudaDeviceSynchronize() != cudaSuccess) return CRK_E_CUDA;
  if (cudaMemcpy(host4, x->ix.ms.stats, 16, cudaMemcpyDeviceToHost) != cudaSuccess) return CRK_E_CUDA;
  return CRK_OK;
}

// Diagnostic (not in the public header): device pointers of the chunked scan's scratch (sums, state, stops,
// plan, log) and its chunk capacity, for inspection tools.
extern "C" int crk_debug_index_ms(crk_index* x, void** ptrs5, uint32_t* chunk_cap) {
  if (!x || !ptrs5 || !chunk_cap) return CRK_E_ARG;
  ptrs5[0] = x->ix.ms.sums;
  ptrs5[1] = x->ix.ms.state;
  ptrs5[2] = x->ix.ms.stops;
  ptrs5[3] = x->ix.ms.plan;
  ptrs5[4] = x->ix.ms.log;
  *chunk_cap = x->ix.ms.chunk_cap;
  return CRK_OK;
}

// Diagnostic (not in the public header): copies the context's 16 scratch counters (crk_internal.h Scratch::
// counters) to host memory after synchronising the device; tests read counters[13] (the mover's run -> job
// map applied) with it.
extern "C" int crk_debug_counters(crk_ctx* c, uint32_t* host16) {
  if (!c || !host16) return CRK_E_ARG;
  DeviceGuard g(c->device);
  if (cudaDeviceSynchronize() != cudaSuccess) return CRK_E_CUDA;
  if (cudaMemcpy(host16, c->sc.counters, 16 * sizeof(uint32_t), cudaMemcpyDeviceToHost) != cudaSuccess)
    return CRK_E_CUDA;
  return CRK_OK;
}

#ifdef CRK_TIMELINE
// Diagnostic build only: kernels of this context stamp [min start, max end] per stage into dev_buf
// (TL_STAGES x 2 u64, device memory; nullptr turns it off).
int crk_debug_timeline(crk_ctx* c, unsigned long long* dev_buf) {
  if (!c) return CRK_E_ARG;
  c->cd.tl = dev_buf;
  return CRK_OK;
}
#endif

struct crk_server {
  crk_ctx* ctx;
  int device;
  cudaStream_t stream;
  crk_server_bell* bell;
  bool host_bell;  // mapped host memory: the CPU writes it directly
  uint32_t n_rings;
};

namespace {
// Writes `stop` and bumps `seq` (CPU stores for a host bell, a copy on a private stream otherwise).
int server_signal(crk_server* S, uint64_t stop) {
  if (S->host_bell) {
    S->bell->stop = stop;
    std::atomic_thread_fence(std::memory_order_seq_cst);
    S->bell->seq = S->bell->seq + 1;
    return CRK_OK;
  }
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  uint64_t seq = 0;
  cudaError_t e = cudaMemcpyAsync(&seq, (const void*)&S->bell->seq, 8, cudaMemcpyDefault, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  seq += 1;
  if (e == cudaSuccess) e = cudaMemcpyAsync((void*)&S->bell->stop, &stop, 8, cudaMemcpyDefault, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e == cudaSuccess) e = cudaMemcpyAsync((void*)&S->bell->seq, &seq, 8, cudaMemcpyDefault, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  cudaStreamDestroy(s);
  return e == cudaSuccess ? CRK_OK : cuda_fail(e);
}
}  // namespace

int crk_server_start(crk_ctx* c, crk_index* x, uint32_t n_rings, const crk_ring* rings, const crk_ring* send_rings,
                     uint64_t region_base, uint64_t region_bytes, crk_server_bell* bell, crk_stream_t stream,
                     crk_server** out) {
  if (!c || !x || x->ctx != c || !rings || !send_rings || !bell || !out) return CRK_E_ARG;
  *out = nullptr;
  if (n_rings == 0 || n_rings > x->ix.max_rings || n_rings > (uint32_t)CRK_MAX_RINGS) return CRK_E_ARG;
  for (uint32_t r = 0; r < n_rings; ++r)
    if (!ring_ok(rings[r]) || !ring_ok(send_rings[r])) return CRK_E_ARG;
  if (x->ix.max_records > crk::server_threads() || 2ull * x->ix.max_records > c->sc.max_jobs) return CRK_E_CAPACITY;
  DeviceGuard g(c->device);
  cudaPointerAttributes a;
  CK(cudaPointerGetAttributes(&a, bell));
  crk_server* S = new (std::nothrow) crk_server;
  if (!S) return CRK_E_CAPACITY;
  S->ctx = c;
  S->device = c->device;
  S->stream = (cudaStream_t)stream;
  S->bell = bell;
  S->host_bell = a.type == cudaMemoryTypeHost;
  S->n_rings = n_rings;
  const cudaError_t e = launch_server(x->ix, c->cd, c->sc, c->d_schemas, bell, n_rings, rings, send_rings,
                                      region_base, region_bytes, S->stream);
  if (e != cudaSuccess) { delete S; return cuda_fail(e); }
  *out = S;
  return CRK_OK;
}

int crk_server_stop(crk_server* S) {
  if (!S) return CRK_E_ARG;
  DeviceGuard g(S->device);
  int st = server_signal(S, 1);
  const cudaError_t e = cudaStreamSynchronize(S->stream);
  delete S;
  if (st != CRK_OK) return st;
  return e == cudaSuccess ? CRK_OK : cuda_fail(e);
}

int crk_server_step(crk_server* S, const uint64_t* heads, const uint64_t* tails, const uint64_t* send_offs,
                    uint64_t timeout_ns) {
  if (!S || !S->host_bell || !heads || !tails || !send_offs) return CRK_E_ARG;
  crk_server_bell* B = S->bell;
  for (uint32_t r = 0; r < S->n_rings; ++r) {
    B->head[r] = heads[r];
    B->tail[r] = tails[r];
    B->send_off[r] = send_offs[r];
  }
  const uint64_t seq = B->seq + 1;
  std::atomic_thread_fence(std::memory_order_release);  // the cursors before seq (x86: stores are ordered)
  B->seq = seq;
  const auto t0 = std::chrono::steady_clock::now();
  for (uint32_t spin = 0; B->done_seq != seq; ++spin) {
    if ((spin & 1023) == 0 &&
        (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(std::chrono::steady_clock::now() - t0).count() >
            timeout_ns)
      return CRK_E_CUDA;
  }
  std::atomic_thread_fence(std::memory_order_acquire);  // results after done_seq
  return B->status;
}

int crk_host_alloc(uint64_t bytes, void** out) {
  if (!out || bytes == 0) return CRK_E_ARG;
  CK(cudaHostAlloc(out, bytes, cudaHostAllocMapped | cudaHostAllocPortable));
  return CRK_OK;
}
void crk_host_free(void* p) {
  if (p) cudaFreeHost(p);
}
int crk_copy_to_host(void* host_dst, const void* dev_src, uint64_t bytes) {
  if (bytes && (!host_dst || !dev_src)) return CRK_E_ARG;
  CK(cudaMemcpy(host_dst, dev_src, bytes, cudaMemcpyDefault));
  return CRK_OK;
}

const char* crk_strerror(int st) {
  switch (st) {
    case CRK_OK: return "ok";
    case CRK_INCOMPLETE: return "incomplete: the window ends inside a record (or the index is full)";
    case CRK_E_ARG: return "bad argument";
    case CRK_E_TRUNCATED: return "item runs past the end of its record";
    case CRK_E_FRAG: return "record longer than max_record_bytes";
    case CRK_E_RPC: return "not an RPC v2 CALL for the configured program/version";
    case CRK_E_AUTH: return "credential or verifier longer than 400 bytes";
    case CRK_E_PAD: return "nonzero XDR pad byte";
    case CRK_E_SIZE: return "size mismatch or count above capacity";
    case CRK_E_TRAILING: return "bytes after the last argument";
    case CRK_E_XID: return "xid not found / duplicate xid";
    case CRK_E_PTR: return "destination too small or outside the registered region";
    case CRK_E_CAPACITY: return "index or scratch capacity exceeded";
    case CRK_E_PROC: return "procedure not registered / not the expected procedure";
    case CRK_E_CUDA: return "CUDA error";
    default: return "unknown status";
  }
}
int crk_profile_enable(int on) {
  if (on && !g_prof.created) {
    for (int s = 0; s < PROF_STAGES; ++s)
      for (int b = 0; b < 2; ++b)
        for (uint32_t i = 0; i < kProfCap; ++i) CK(cudaEventCreate(&g_prof.ev[s][b][i]));
    g_prof.created = true;
  }
  g_prof.on = on != 0;
  for (int s = 0; s < PROF_STAGES; ++s) g_prof.n[s] = 0;
  return CRK_OK;
}

int crk_profile_read(double* ms, uint32_t* launches) {
  if (!ms || !launches) return CRK_E_ARG;
  for (int s = 0; s < PROF_STAGES; ++s) {
    double acc = 0;
    for (uint32_t i = 0; i < g_prof.n[s]; ++i) {
      float t = 0;
      CK(cudaEventSynchronize(g_prof.ev[s][1][i]));
      CK(cudaEventElapsedTime(&t, g_prof.ev[s][0][i], g_prof.ev[s][1][i]));
      acc += t;
    }
    ms[s] = acc;
    launches[s] = g_prof.n[s];
    g_prof.n[s] = 0;
  }
  return CRK_OK;
}

int crk_last_cuda_error(void) { return g_last_cuda; }
int crk_kernel_launches(void) { return crk::g_launches.load(); }
const char* crk_version(void) { return "crk 0.1 (sm_100a)"; }

}  // extern "C"
