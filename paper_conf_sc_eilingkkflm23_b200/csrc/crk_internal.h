// Internal structures shared by the crk kernels and the C ABI layer (not part of the public ABI).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/crk.h"

namespace crk {

constexpr int kMaxItems = CRK_MAX_ITEMS;
constexpr int kMaxProcs = CRK_MAX_PROCS;
constexpr int kMaxRings = CRK_MAX_RINGS;
constexpr int kScanThreads = 1024;  // K1: one CTA per ring, one candidate header per thread
constexpr int kParseWarps = 4;      // K3: one warp per record (small CTAs co-reside with the mover)
constexpr int kMoveThreads = 256;   // K4/K6 mover CTA
constexpr int kMaxPieces = 2 * kMaxItems + 2;

struct Schema {
  uint32_t proc, n_items;
  uint32_t items[kMaxItems];
};
struct SchemaTable {
  uint32_t n;
  Schema s[kMaxProcs];
};

struct RingDesc {
  uint8_t* base;
  uint64_t mask;  // cap - 1
  uint64_t head, tail;
};

// ---- chunked scan of long windows (k_mscan.cu): per-index scratch --------------------------------
constexpr uint32_t kCand = 4;       // candidate chains walked per chunk
constexpr uint32_t kLogCap = 512;   // headers logged per chain
struct alignas(16) ChainSum {       // one candidate chain of one chunk (64 bytes)
  uint64_t start, exit;             // its first header; the cursor after its last logged header
  uint64_t r0_after, sum_after;     // after its last last-fragment header: next record start, lengths since
  uint64_t sum_total;               // sum of all logged lengths
  uint32_t n, nlast;                // logged headers, of which last fragments
  int32_t idx_last;                 // log index of the last last-fragment header (-1: none)
  uint32_t kind;                    // CH_* (k_mscan.cu)
  uint64_t pad_;
};
static_assert(sizeof(ChainSum) == 64, "ChainSum is read as four 16-byte words");
struct ChunkState {                 // the walk state at a chunk's true entry (written by the resolver)
  uint64_t p, r0, sum;
  uint32_t nf, nr, f0;
  int32_t chosen;                   // candidate chain holding the true chain, -1: no header starts here
  uint32_t skip;                    // log entries of that chain before the true entry (a false start fed it)
  uint32_t pad_;
};
struct ChunkStop {                  // outcome of a check that failed in this chunk's emission
  uint64_t consumed;
  int32_t status;
  uint32_t nr, kept, pad_;
};
struct RingPlan {                   // per ring of the index
  uint32_t ticket_a, ticket_b, fallback, pad_;
  unsigned long long stop_key;      // min over failing hops of (fragment number << 24 | chunk), ~0 = none
  crk_ring_result end;              // the outcome when no check fails (end of the chain)
};
struct MultiScanDev {
  uint32_t chunk_cap;               // chunks one launch can hold
  uint2* log;                       // [chunk_cap * kCand * kLogCap]: (cursor - chunk start, header)
  ChainSum* sums;                   // [chunk_cap * kCand]
  ChunkState* state;                // [chunk_cap]
  ChunkStop* stops;                 // [chunk_cap]
  RingPlan* plan;                   // [max_rings]
  uint32_t* stats;                  // [4] diagnostic totals: rings resolved chunked, rings that fell back
};

// One parent memcpy of a serve step's striped HtoD CALLs (reading R22).  Open addressing by parent xid over
// a table that is all ~0 between steps (the planner resets the entries it used): key = parent xid; ptr / total
// claimed by the first OK stripe (CAS from ~0), good cleared by a stripe that disagrees; landed_c = ~(bytes
// landed); lead = the smallest dense id of an OK stripe at offset 0.
struct StripeEnt {                  // 48 bytes
  unsigned long long key, ptr, total, landed_c;
  uint32_t lead, good;
  unsigned long long pad_;
};

// Device-resident tables of one index (pointers into one cudaMalloc block).
struct IndexDev {
  uint32_t max_rings, frags_per_ring, recs_per_ring, max_records;
  uint32_t hash_mask;
  RingDesc* rings;              // [max_rings]
  crk_ring_result* res;         // [max_rings]
  uint32_t* rec_prefix;         // [max_rings + 1]; [n_rings] = total
  uint32_t* total;              // device scalar (== rec_prefix[n_rings])
  uint32_t* ticket;             // scan finish ticket
  uint64_t* frag_phys;
  uint64_t* frag_lstart;
  uint32_t* frag_hdr;
  uint64_t* rec_begin;
  uint64_t* rec_len;
  uint32_t* rec_frag0;
  uint32_t* rec_nfrags;
  uint32_t* p_slot;
  uint32_t* p_ring;
  uint32_t* p_xid;
  uint32_t* p_proc;
  int32_t* p_status;
  uint32_t* p_nitems;
  uint32_t* p_frag0;            // the record's first fragment (absolute), fragment count, first fragment's length:
  uint32_t* p_nfrags;           // written by the parser, so a decode job is built without the chain of
  uint32_t* p_flen0;            // slot -> record table -> fragment table loads
  uint32_t* p_kind;
  uint64_t* p_off;
  uint64_t* p_count;
  uint64_t* p_value;
  int32_t* s_status;
  int32_t* s_reply_err;
  uint64_t* s_reply_off;
  uint64_t* s_reply_wire;
  unsigned long long* xid_hash;  // (xid << 32 | dense id), empty = ~0
  MultiScanDev ms;               // chunked scan scratch
  StripeEnt* stripe;             // [hash_mask + 1] parent memcpys of the step (reading R22)
  uint32_t* stripe_list;         // [max_records] table slots in use
  uint32_t* stripe_n;            // [2]: slots in use, planning-pass ticket
};

// ---- mover jobs ----------------------------------------------------------------------------------
// Decode: dst[0..nbytes) <- logical bytes [loff, loff + nbytes) of record `rec`, element-swapped by esize.
// Encode: the framed record whose logical bytes are the pieces is written to ring `out` from cursor.
enum : uint32_t { JOB_NONE = 0, JOB_DEC = 1, JOB_ENC = 2 };
enum : uint32_t { PIECE_WORDS = 0, PIECE_DATA = 1 };

struct Piece {            // 64 bytes
  uint64_t loff;          // logical offset of the piece within the record
  uint64_t nbytes;        // WORDS: 4 * nwords; DATA: payload bytes (zero pad to 4 follows implicitly)
  uint64_t src;           // DATA: device address of element 0
  uint32_t esize;         // DATA: 1, 4 or 8
  uint32_t type;          // PIECE_WORDS / PIECE_DATA
  uint32_t words[8];      // WORDS: host-order values written big-endian
};

struct Job {              // 64 bytes
  uint32_t type;          // JOB_*
  uint32_t esize;         // DEC: element size
  uint32_t rec;           // DEC: dense record id
  uint32_t n_pieces;      // ENC: pieces; DEC: the record's fragment count
  uint64_t out_start;     // DEC: dst address; ENC: out-ring cursor of the record's first header byte
  uint64_t out_end;       // exclusive (DEC: dst + nbytes; ENC: out_start + wire size)
  uint64_t loff;          // DEC: logical offset of the first byte; ENC: logical length of the record
  uint32_t piece0;        // ENC: first piece in the piece pool; DEC: the record's first fragment (absolute)
  uint32_t F;             // ENC: fragment payload (0 -> explicit fragment table); DEC: first fragment's length
  uint32_t lens0;         // ENC with explicit framing: first entry in the lens / wire-start pool
  uint32_t n_lens;
  uint32_t out_ring;      // ENC: index into the out-ring table; DEC: the record's ring
  uint32_t pad_;
};

struct Scratch {          // ctx-owned device scratch
  Job* jobs;              // [max_jobs]
  Piece* pieces;          // [2 * max_jobs]
  uint32_t* counters;     // [16]: 0/2 mover decode/encode run cursors, 3/6 their single-tile tail cursors, 1 n_jobs,
                          // 15 the fused front end's lean back-off (steps left before the lean path is tried again),
                          // 4 queue split, 5 K2 block counter, 8/9 mover launch stamp (sequence, start time),
                          // 12 queue-0 runs in run_job, 13 run_job valid for the next mover launch
  uint64_t* lens_pool;    // explicit framing: [2 * max_lens] (lens, then wire starts)
  uint32_t* lens32;       // [max_lens] staging for host-given fragment lengths
  unsigned long long* scan_state;  // decoupled look-back state for K2
  uint64_t* scan_tmp;     // [max_jobs + 2]: sizes -> prefix; [max_jobs + 1] = total
  RingDesc* out_rings;    // [kMaxRings]
  uint32_t* run_job;      // [max_jobs]: the job holding each mover run's first tile (queue 0 runs, then queue 1)
  uint32_t max_jobs, max_lens, max_pieces;
  uint32_t mover_seq;     // host-side count of this context's mover launches (the launch stamp's sequence)
  uint32_t pdl;           // launches with programmatic dependent launch (see launch_k)
};

struct ConfigDev {
  uint32_t F, strict, prog, vers, proc_h2d, proc_d2h, guess, tile_shift;
  uint32_t scan_threads, stages, run, tail;  // tail: per-CTA single-tile claims at the end of each queue
  uint32_t reserve;         // mover CTAs that run only when the launch found the GPU free (crk_config.mover_reserve_ctas)
  uint32_t no_chunked_scan; // crk_config.scan_chunking == 1: one CTA per ring always
  uint32_t proc_stripe;     // crk_config.proc_h2d_stripe (0: none)
  uint32_t lean;            // crk_config.lean_steps
  uint32_t lean_backoff;    // crk_config.lean_backoff
  uint32_t pad3_;
  uint64_t max_record_bytes;
  unsigned long long* tl;  // diagnostic timeline build only (-DCRK_TIMELINE): [stage][min start, max end]
};

// ---- launchers (defined in the k_*.cu files) ------------------------------------------------------
struct ScanRingsParam {
  uint32_t n_rings;
  RingDesc r[kMaxRings];
  // optional: cursors read at execution time (device or mapped memory, u64 [heads n | tails n | send offs n]);
  // lets a captured serve graph be replayed as the rings advance
  const uint64_t* doorbell;
};

cudaError_t launch_frame_scan(const IndexDev& ix, const ScanRingsParam& p, const ConfigDev& cfg, cudaStream_t s);
// Chunked multi-CTA scan of long windows (k_mscan.cu): chunk_plan fills an opaque parameter block
// (chunk_param_bytes()) and returns false when every ring is short enough for the one-CTA scan.
bool chunk_plan(const IndexDev& ix, const ScanRingsParam& p, int sms, void* out_param);
size_t chunk_param_bytes();
uint32_t chunk_plan_chunks(const void* param);
cudaError_t launch_chunk_scan(const IndexDev& ix, const void* param, const ConfigDev& cfg, cudaStream_t s);
cudaError_t launch_parse(const IndexDev& ix, const SchemaTable* schemas, const ConfigDev& cfg, uint32_t n_rings,
                         int sms, cudaStream_t s);
// Exclusive scan of n u64 values in place; total (may be null) gets the sum.  n read from n_dev if
// n_dev is non-null (device count), else n.
cudaError_t launch_exclusive_scan_u64(uint64_t* data, uint32_t n, const uint32_t* n_dev, uint64_t* total,
                                      Scratch& sc, cudaStream_t s);
cudaError_t launch_exclusive_scan_u32(uint32_t* data, uint32_t n, const uint32_t* n_dev, uint32_t* total,
                                      Scratch& sc, cudaStream_t s);

// Resolving requests into jobs.
struct H2DReq {
  uint32_t xid;
  void* dst;
  uint64_t dst_bytes;
  int32_t* status;
  uint64_t* copied;
};
cudaError_t launch_resolve_h2d(const IndexDev& ix, const ConfigDev& cfg, Scratch& sc, uint32_t n, const uint32_t* xids,
                               void* const* dsts, const uint64_t* dst_bytes, int32_t* statuses, uint64_t* copied,
                               const H2DReq* single, cudaStream_t s);
cudaError_t launch_resolve_items(const IndexDev& ix, const ConfigDev& cfg, Scratch& sc, uint32_t n,
                                 const crk_item_req* reqs, const crk_item_req* single, cudaStream_t s);
cudaError_t launch_serve_plan(const IndexDev& ix, const ConfigDev& cfg, Scratch& sc, uint32_t n_rings,
                              const crk_ring* send_rings, const uint64_t* send_offs, uint64_t region_base,
                              uint64_t region_bytes, const uint64_t* doorbell, cudaStream_t s);
// Encode jobs built on the host (<= a few per call) are copied in by value.
struct EncJobParam {
  uint32_t n_jobs, n_pieces;
  Job jobs[2];
  Piece pieces[kMaxPieces];
};
// One job (n_jobs == 1) is planned in place: the mover follows directly (launch_plan_and_move planned=true).
cudaError_t launch_put_enc_jobs(Scratch& sc, const ConfigDev& cfg, const EncJobParam& p, const RingDesc& out,
                                cudaStream_t s);
cudaError_t launch_d2h_batch_jobs(Scratch& sc, const ConfigDev& cfg, uint32_t n, const uint32_t* xids,
                                  const void* const* srcs, const uint64_t* bytes, const int32_t* errs,
                                  const RingDesc& out, uint64_t out_off, uint64_t* wire_offs, uint64_t* total,
                                  cudaStream_t s);
cudaError_t launch_put_lens(Scratch& sc, const uint32_t* lens32_dev, uint32_t n, cudaStream_t s);
cudaError_t launch_replies_jobs(Scratch& sc, const ConfigDev& cfg, uint32_t n, const crk_reply_req* reqs,
                                const RingDesc& out, uint64_t out_off, uint64_t* wire_offs, uint64_t* total,
                                cudaStream_t s);
// Plans tiles for jobs [0, n_jobs) (n_jobs from counters[1] <= max_jobs_bound) and runs the mover.
// out_bytes_bound (0 = unknown) caps the mover grid for small requests.
// planned: the jobs' tile prefix and cursors were already written (single-request kernels).
cudaError_t launch_plan_and_move(const IndexDev* ix, const ConfigDev& cfg, Scratch& sc, uint32_t max_jobs_bound,
                                 uint64_t out_bytes_bound, int sms, int move_ctas, cudaStream_t s,
                                 bool planned = false);
int mover_occupancy(uint32_t tile_bytes, uint32_t stages);
constexpr int kMaxDevices = 64;
cudaError_t ensure_mover_smem(uint32_t smem);  // per-device dynamic shared memory opt-in, raise-only
cudaError_t launch_mover(const IndexDev* ix, const ConfigDev& cfg, Scratch& sc, uint32_t run, int move_ctas,
                         cudaStream_t s, bool use_map = false);
// Serve planning for small batches (index max_records <= kSmallServe): statuses, reply offsets, decode
// and encode jobs, their tile prefix and the mover cursors in one single-block kernel.
constexpr uint32_t kSmallServe = 1024;
cudaError_t launch_serve_plan_small(const IndexDev& ix, const ConfigDev& cfg, Scratch& sc, uint32_t n_rings,
                                    const crk_ring* send_rings, const uint64_t* send_offs, uint64_t region_base,
                                    uint64_t region_bytes, const uint64_t* doorbell, cudaStream_t s);

// Fused front end for small serve steps (k_front.cu): scan + parse + plan_small_block in one CTA; the
// mover (launch_mover) follows.  rings: validated scan parameters (cursors or doorbell).
uint32_t front_small_threads();
cudaError_t launch_front_small(const IndexDev& ix, const ConfigDev& cfg, Scratch& sc, const SchemaTable* schemas,
                               const ScanRingsParam& rings, uint32_t n_rings, const crk_ring* send_rings,
                               const uint64_t* send_offs, uint64_t region_base, uint64_t region_bytes,
                               const uint64_t* doorbell, bool plan, cudaStream_t s);

// Persistent server (k_server.cu): one resident CTA of server_threads() threads.
uint32_t server_threads();
cudaError_t launch_server(const IndexDev& ix, const ConfigDev& cfg, const Scratch& sc, const SchemaTable* schemas,
                          crk_server_bell* bell, uint32_t n_rings, const crk_ring* rings, const crk_ring* send_rings,
                          uint64_t region_base, uint64_t region_bytes, cudaStream_t s);

// host-visible counter of our kernel launches
void count_launch(int n = 1);

// Every library kernel is launched with programmatic stream serialization (PDL): it may be scheduled while
// the stream's previous kernel is still running and waits for it in pdl_entry() (crk_device.cuh).
// pdl = false launches it as an ordinary stream-ordered kernel (its pdl_entry() waits for nothing).
template <typename... KArgs, typename... Args>
cudaError_t launch_k_opt(bool pdl, void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                         Args&&... args) {
  cudaLaunchConfig_t c = {};
  c.gridDim = grid;
  c.blockDim = block;
  c.dynamicSmemBytes = smem;
  c.stream = s;
  cudaLaunchAttribute a[1];
  a[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  a[0].val.programmaticStreamSerializationAllowed = 1;
  c.attrs = a;
  c.numAttrs = pdl ? 1 : 0;
  count_launch();
  return cudaLaunchKernelEx(&c, kernel, static_cast<KArgs>(args)...);
}
// Launches a kernel through launch_k_opt; returns its error from the calling launcher.
#define CRK_LAUNCH(...)                            \
  do {                                             \
    const cudaError_t le_ = launch_k_opt(__VA_ARGS__); \
    if (le_ != cudaSuccess) return le_;            \
  } while (0)

// A context launches this way unless it keeps reserved mover CTAs (crk_config.mover_reserve_ctas > 0: a
// pipelined server loop with batches in flight on several streams): there, kernels resident early would sit on
// the SM slots the other batches' kernels need (measured: C5 step 0.347 -> 0.371 ms), while a lone call saves
// each launch gap (C3 4 KiB HtoD call 31 -> 21 us).
__host__ __device__ inline bool pdl_of(const ConfigDev& cfg) { return cfg.reserve == 0; }

// optional CUDA-event timing of the pipeline stages (crk_profile_*)
enum { PROF_SCAN = 0, PROF_PARSE = 1, PROF_PLAN = 2, PROF_MOVE = 3, PROF_STAGES = 4 };
void prof_mark(int stage, bool begin, cudaStream_t s);

}  // namespace crk
