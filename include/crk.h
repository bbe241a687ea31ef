/*
 * crk.h — C ABI of the B200-native server data path for Cricket's RPC-forwarded cudaMemcpy.
 *
 * What it computes.  Cricket forwards CUDA API calls as ONC RPCs (§3.3/§3.5;
 * ONC RPC = RFC 5531, §3.4).  Large memcpy arguments travel as fragmented records
 * (§2) over the RPC connection, and the server "receives the data in a buffer and
 * transfers it to the GPU" (§4.2).  This library is that server data path on the GPU:
 *   - record marking (RFC 5531 §11): 4-byte header, bit 31 = last fragment, bits 0-30 = length;
 *   - the CALL header (RFC 5531 §9, opaque_auth §8.2) and the XDR arguments (RFC 4506): opaque<>
 *     with zero padding (§4.9-4.10), big-endian int/unsigned/hyper/float/double and their arrays
 *     (§4.1-4.7, §4.12-4.13);
 *   - the REPLY (RFC 5531 §9) carrying memcpy DtoH data, framed back into a send ring.
 * Every byte is moved by hand-written sm_100a kernels; the exact byte semantics (and every point the
 * paper leaves open) are DESIGN.md §3-§4, mirrored by the independent CPU oracle in oracle/.
 *
 * Memory model.
 *   - A ring (crk_ring) is caller-owned bytes, either device memory or pinned host memory that is
 *     mapped into the device's address space (cudaHostAlloc / cudaHostRegister with UVA; the host
 *     pointer is used directly, zero-copy over PCIe).  base must be 256-byte aligned, cap a power of
 *     two >= 256.  Positions are unmasked 64-bit cursors; byte c lives at base[c & (cap - 1)].
 *   - Destinations / sources named by calls are device memory (or mapped host memory).
 *   - The context owns scratch only, allocated at create; no call allocates memory.
 *   - "dev" output pointers below may be device memory or mapped pinned host memory; they are
 *     written by kernels and valid once `stream` has completed.
 *
 * Errors.  Every entry point returns an int32 status.  Host-argument errors (CRK_E_ARG) and launch
 * failures (CRK_E_CUDA, see crk_last_cuda_error) are returned synchronously.  Data-dependent statuses
 * are written asynchronously to the status slots named by each call.  On any data error the
 * destination is left untouched: all checks precede the bulk write (reading R17).
 * Calls on one crk_index must be ordered on one stream; different indexes may run concurrently.
 */
#ifndef CRK_H
#define CRK_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* cudaStream_t without pulling in cuda_runtime.h */
typedef struct CUstream_st* crk_stream_t;

/* ---- status codes ---- */
#define CRK_OK 0
#define CRK_INCOMPLETE 1      /* window ends inside a record / index full: call again with more bytes */
#define CRK_E_ARG (-1)        /* bad host argument, or argument kind mismatch (typed decode) */
#define CRK_E_TRUNCATED (-2)  /* an item runs past the end of its record */
#define CRK_E_FRAG (-3)       /* record longer than max_record_bytes */
#define CRK_E_RPC (-4)        /* msg_type != CALL, rpcvers != 2, or prog/vers not the configured ones */
#define CRK_E_AUTH (-5)       /* cred or verf body longer than 400 bytes (RFC 5531 §8.2) */
#define CRK_E_PAD (-6)        /* nonzero XDR pad byte (strict mode) */
#define CRK_E_SIZE (-7)       /* opaque length != size argument (strict), or count > caller capacity */
#define CRK_E_TRAILING (-8)   /* bytes after the last argument (strict mode) */
#define CRK_E_XID (-9)        /* xid not in the index / a later duplicate of an earlier record's xid */
#define CRK_E_PTR (-10)       /* destination too small / pointer outside the registered region */
#define CRK_E_CAPACITY (-11)  /* index or scratch too small for even one record / the request */
#define CRK_E_PROC (-12)      /* procedure has no registered schema / record is not of the expected proc */
#define CRK_E_CUDA (-100)     /* CUDA runtime error */

/* ---- XDR item kinds of an argument schema; fixed-length kinds carry their count in bits 8..31 ---- */
#define CRK_K_U32 1         /* int / unsigned int / enum / bool (RFC 4506 §4.1-4.4) */
#define CRK_K_U64 2         /* hyper / unsigned hyper (§4.5) */
#define CRK_K_OPAQUE_VAR 3  /* opaque<> and string<> (§4.10, §4.11) */
#define CRK_K_OPAQUE_FIX 4  /* opaque[n] (§4.9) */
#define CRK_K_I32_VAR 5     /* int<> (§4.13) */
#define CRK_K_U32_VAR 6
#define CRK_K_F32_VAR 7     /* float<> (§4.6) */
#define CRK_K_I64_VAR 8     /* hyper<> */
#define CRK_K_U64_VAR 9
#define CRK_K_F64_VAR 10    /* double<> (§4.7) */
#define CRK_K_I32_FIX 11    /* int[n] (§4.12) */
#define CRK_K_U32_FIX 12
#define CRK_K_F32_FIX 13
#define CRK_K_I64_FIX 14
#define CRK_K_U64_FIX 15
#define CRK_K_F64_FIX 16
#define CRK_ITEM(kind, fixed_count) ((uint32_t)(kind) | ((uint32_t)(fixed_count) << 8))
#define CRK_MAX_ITEMS 8
#define CRK_MAX_PROCS 64
#define CRK_MAX_RINGS 64

typedef struct {
  uint8_t* base; /* device pointer or mapped pinned host pointer, 256-byte aligned */
  uint64_t cap;  /* power of two >= 256 */
} crk_ring;

typedef struct {
  uint32_t frag_payload;     /* F: data bytes per fragment when encoding (default 65536, reading R4) */
  int32_t strict;            /* 1 (default): E_PAD / E_TRAILING / E_SIZE checks on; 0: lenient (reading R5, R9) */
  uint64_t max_record_bytes; /* records longer than this fail with E_FRAG (default 2^32) */
  uint32_t prog, vers;       /* RPC program / version accepted by the decoder (reading R15) */
  uint32_t proc_h2d;         /* built-in schema (ptr u64, mem opaque<>, size u64) */
  uint32_t proc_d2h;         /* built-in schema (ptr u64, size u64) */
  uint32_t scan_stride_guess;/* first stride the speculative scanner tries (default frag_payload) */
  uint32_t tile_bytes;       /* bytes per mover work tile, power of two in [1024, 1<<20] (default 32768) */
  uint32_t max_jobs;         /* decode + encode job capacity per call (default 1<<20) */
  uint32_t ctas_per_sm;      /* mover occupancy override, 0 = occupancy calculator */
  uint32_t scan_threads;     /* K1 threads per ring, two predictor groups, 64..1024, multiple of 64 (default 256) */
  uint32_t mover_stages;     /* mover pipeline stages, 2..8 (default 3) */
  uint32_t mover_run;        /* tiles per mover claim, 1..64 (default 8) */
  uint32_t mover_tail_tiles; /* per mover CTA, the last tiles of each queue claimed one at a time, 0..64 (default 2;
                                shortens the kernel's tail when it runs alone) */
  uint32_t mover_reserve_ctas; /* opportunistic mover CTAs (default 0, < half the grid): the last N CTAs of a
                                  mover launch run only if they start within 10 us of its first CTA (the GPU was
                                  free: a lone call gets the whole grid); behind another batch's mover (several
                                  batches in flight on other streams) they exit at once, so the next batch's
                                  scan / parse / plan kernels find room on the GPU while this mover streams */
  uint32_t fused_front_max_records; /* crk_serve with an index of at most this many records (and at most
                                       fused_front_max_window bytes of ring windows; with scan_chunking = 1 also
                                       any single ring) runs scan + parse + planning as ONE single-CTA launch
                                       before the mover (default 128, at most 1024 takes effect; 0 = always
                                       separate kernels) */
  uint32_t scan_chunking;    /* 0 (default): windows of at least 2 chunks (>= 512 KiB) are scanned by the chunked
                                multi-CTA scan (one CTA per chunk); 1: always one CTA per ring */
  uint64_t fused_front_max_window; /* default 1 MiB (one CTA scans the rings in turn) */
  uint32_t proc_h2d_stripe;  /* built-in schema (ptr u64, mem opaque<>, size u64, parent u32, offset u64, total u64):
                                one stripe of a memcpy sent over several connections (reading R22;
                                default 3, 0 = no such procedure) */
  uint32_t mover_max_ctas;    /* cap on the mover's grid (0 = every CTA slot the occupancy allows); a small grid
                                leaves HBM to concurrent copy-engine traffic in a host-ring server loop */
  uint32_t fused_front_max_frags; /* a small index (fused_front_max_records) whose rings hold at most this many
                                     fragments in all also takes the fused single-CTA front end for windows past
                                     fused_front_max_window: the index bounds the CTA's header walk (default
                                     4096, e.g. one 256 MiB memcpy CALL in 64 KiB fragments; 0 = off) */
  uint32_t lean_steps;       /* 1 (default): a persistent-server or fused crk_serve step of well-formed memcpy CALLs
                                (AUTH_NONE, built-in HtoD / DtoH procedures, distinct xids, all served OK, <= 32
                                records / 64 KiB of windows and of DtoH replies) is served by one warp over a
                                shared-memory copy of the windows (DESIGN.md §1 item 22; identical results); any
                                other step runs the general phases.  0: always the general phases */
  uint32_t lean_backoff;     /* steps that skip the lean attempt after a step it could not take (default 16;
                                0: try every step) */
} crk_config;

typedef struct crk_ctx crk_ctx;
typedef struct crk_index crk_index;

/* Per-ring result of a scan or serve call (written to the index; read with crk_index_ring_results). */
typedef struct {
  int32_t status;       /* OK, INCOMPLETE, E_FRAG, E_CAPACITY (first failing check) */
  uint32_t n_records;   /* complete records indexed for this ring */
  uint32_t n_frags;     /* their fragments */
  uint32_t rec_base;    /* dense id of this ring's first record */
  uint64_t consumed;    /* cursor of the first byte not consumed (start of the first incomplete record) */
  uint64_t reply_bytes; /* serve only: wire bytes of replies appended to this ring's send ring */
} crk_ring_result;

/* Device pointers into an index (for inspection and tests).  Fragment and record tables are laid out
 * in per-ring slices: ring r's fragments start at r * frags_per_ring, its records at r * recs_per_ring.
 * Parsed tables are dense: record d (0 .. total) of ring r is d - rec_base[r] within its slice. */
typedef struct {
  uint32_t max_rings, frags_per_ring, recs_per_ring, max_records;
  /* fragments (slice layout) */
  uint64_t* frag_phys;    /* cursor of the fragment's first data byte */
  uint64_t* frag_lstart;  /* logical offset of that byte within its record */
  uint32_t* frag_hdr;     /* the raw header: length | last << 31 */
  /* records (slice layout) */
  uint64_t* rec_begin;    /* cursor of the record's first header */
  uint64_t* rec_len;      /* logical length */
  uint32_t* rec_frag0;    /* absolute index of its first fragment */
  uint32_t* rec_nfrags;
  /* parsed CALLs (dense) */
  uint32_t* p_slot;       /* slice index of dense record d */
  uint32_t* p_ring;
  uint32_t* p_xid;
  uint32_t* p_proc;
  int32_t* p_status;      /* wire-level status (parse incl. strict trailing check) */
  uint32_t* p_nitems;
  uint32_t* p_kind;       /* [d * CRK_MAX_ITEMS + i] */
  uint64_t* p_off;        /* logical offset of item i's data (after its count word) */
  uint64_t* p_count;      /* opaque bytes / array elements */
  uint64_t* p_value;      /* U32/U64 scalar value */
  int32_t* serve_status;  /* serve only: final per-record status (wire, E_XID, E_SIZE, E_PTR) */
  int32_t* serve_reply_err;/* serve only: -1 no reply, 0 / 1 the mem_result discriminant */
  uint64_t* serve_reply_off;/* serve only: send-ring cursor of the reply (0 when the record has none) */
  uint64_t* serve_reply_wire;
  crk_ring_result* ring_results; /* [max_rings] */
  uint32_t* total_records;       /* device scalar */
} crk_index_view;

/* ---------------------------------------------------------------- setup (control path) */
void crk_config_init(crk_config* cfg);
int crk_ctx_create(int device, const crk_config* cfg, crk_ctx** out);
void crk_ctx_destroy(crk_ctx* ctx);
/* Registers an argument schema for `proc` (items: CRK_ITEM codes, n <= CRK_MAX_ITEMS).  The built-in
 * memcpy schemas for cfg.proc_h2d / proc_d2h are registered at create.  Synchronous. */
int crk_proc_schema_register(crk_ctx* ctx, uint32_t proc, const uint32_t* items, uint32_t n);
/* An index holds the fragment/record/parse tables of up to max_rings rings; each ring gets an equal
 * slice (max_frags / max_rings fragments, max_records / max_rings records). */
int crk_index_create(crk_ctx* ctx, uint32_t max_rings, uint32_t max_frags, uint32_t max_records, crk_index** out);
void crk_index_destroy(crk_index* idx);
int crk_index_get_view(const crk_index* idx, crk_index_view* out);
/* Copies the per-ring results of the last scan/serve to host memory and waits for `stream`. */
int crk_index_ring_results(crk_index* idx, uint32_t n_rings, crk_ring_result* host_out, crk_stream_t stream);
/* The same copy without waiting: `pinned_out` must be pinned host memory; valid once `stream` completes. */
int crk_index_ring_results_async(crk_index* idx, uint32_t n_rings, crk_ring_result* pinned_out, crk_stream_t stream);

/* Copies the cursor window [head, tail) of ring `src` into ring `dst` at the same cursors (each side
 * wrapping at its own capacity) with copy-engine DMA (cudaMemcpyAsync, any direction).  This is the
 * staging step of the copy-engine e2e mode: a pinned host receive ring is moved into a device ring that
 * crk_serve then reads from HBM, and reply bytes are moved back out of a device send ring.
 * tail - head must not exceed either capacity. */
int crk_ring_copy(crk_ring dst, crk_ring src, uint64_t head, uint64_t tail, crk_stream_t stream);

/* ---------------------------------------------------------------- K1-K3: frame scan + CALL parse
 * Scans ring r's window [heads[r], tails[r]) (RFC 5531 §11), fills the fragment table with each
 * fragment's cursor, length and logical start (segmented prefix sum over fragment lengths), then
 * parses every complete record as a CALL (RFC 5531 §9 + the proc's schema, RFC 4506) and builds the
 * xid lookup (earliest record owns an xid, reading R11).  Per-ring results: crk_index_ring_results.
 * n_rings <= min(CRK_MAX_RINGS, the index's max_rings); heads/tails are host arrays. */
int crk_rpc_frame_scan(crk_ctx* ctx, crk_index* idx, uint32_t n_rings, const crk_ring* rings,
                       const uint64_t* heads, const uint64_t* tails, crk_stream_t stream);

/* ---------------------------------------------------------------- K4: memcpy HtoD decode
 * The record owning `xid` must be a proc_h2d CALL (ptr u64, mem opaque<>, size u64).  Checks in order
 * (DESIGN.md §4): its wire status; E_PROC; E_SIZE (strict, mem.n != size); E_PTR (dst_bytes < n).
 * Then dst[0..n) = the opaque payload gathered across fragments; nothing else is written.
 * status_dev / copied_dev: dev int32 / uint64 slots (copied_dev may be NULL). */
int crk_xdr_decode_memcpy_h2d(crk_ctx* ctx, crk_index* idx, uint32_t xid, void* dst, uint64_t dst_bytes,
                              int32_t* status_dev, uint64_t* copied_dev, crk_stream_t stream);
/* n requests at once; xids, dsts, dst_bytes, statuses, copied are dev arrays of length n.  A request whose
 * checks pass but whose dst is NULL with a non-empty payload gets CRK_E_ARG (after E_PTR) and copies nothing. */
int crk_xdr_decode_memcpy_h2d_batch(crk_ctx* ctx, crk_index* idx, uint32_t n, const uint32_t* xids,
                                    void* const* dsts, const uint64_t* dst_bytes, int32_t* statuses,
                                    uint64_t* copied, crk_stream_t stream);

/* ---------------------------------------------------------------- K5: typed / opaque argument decode
 * Argument arg_no of the record owning `xid`, which must be of the named kind (E_ARG otherwise);
 * count > max_count -> E_SIZE.  dst[i] = element i converted from big-endian (floats as bit patterns,
 * reading R13).  dst must be aligned to the element size. */
int crk_xdr_decode_array_i32(crk_ctx*, crk_index*, uint32_t xid, uint32_t arg_no, int32_t* dst, uint64_t max_count,
                             uint64_t* count_dev, int32_t* status_dev, crk_stream_t);
int crk_xdr_decode_array_u32(crk_ctx*, crk_index*, uint32_t xid, uint32_t arg_no, uint32_t* dst, uint64_t max_count,
                             uint64_t* count_dev, int32_t* status_dev, crk_stream_t);
int crk_xdr_decode_array_i64(crk_ctx*, crk_index*, uint32_t xid, uint32_t arg_no, int64_t* dst, uint64_t max_count,
                             uint64_t* count_dev, int32_t* status_dev, crk_stream_t);
int crk_xdr_decode_array_u64(crk_ctx*, crk_index*, uint32_t xid, uint32_t arg_no, uint64_t* dst, uint64_t max_count,
                             uint64_t* count_dev, int32_t* status_dev, crk_stream_t);
int crk_xdr_decode_array_f32(crk_ctx*, crk_index*, uint32_t xid, uint32_t arg_no, float* dst, uint64_t max_count,
                             uint64_t* count_dev, int32_t* status_dev, crk_stream_t);
int crk_xdr_decode_array_f64(crk_ctx*, crk_index*, uint32_t xid, uint32_t arg_no, double* dst, uint64_t max_count,
                             uint64_t* count_dev, int32_t* status_dev, crk_stream_t);
/* opaque<> / opaque[n] argument: max_count is dst capacity in bytes; count_dev receives the length. */
int crk_xdr_decode_opaque(crk_ctx*, crk_index*, uint32_t xid, uint32_t arg_no, void* dst, uint64_t max_count,
                          uint64_t* count_dev, int32_t* status_dev, crk_stream_t);

/* Generic batch: one request per element (device array of n).  Per-request checks in order: E_XID, wire
 * status, E_ARG (arg_no / kind), E_SIZE (count > max_count), then E_ARG for a NULL dst with count > 0 or a
 * dst not aligned to the element size (the single-request calls reject those synchronously). */
typedef struct {
  uint32_t xid, arg_no, kind, pad_;
  void* dst;
  uint64_t max_count;
  uint64_t* count;   /* dev slot or NULL */
  int32_t* status;   /* dev slot */
} crk_item_req;
int crk_xdr_decode_items_batch(crk_ctx* ctx, crk_index* idx, uint32_t n, const crk_item_req* reqs_dev,
                               crk_stream_t stream);

/* ---------------------------------------------------------------- K6/K7: encode
 * Wire size of a memcpy DtoH reply of `bytes` payload with fragment payload F (closed form):
 *   logical = 24 (REPLY header) + 4 (err) + [err == 0: 4 + bytes + pad(bytes)], wire = logical + 4 * max(1, ceil(logical / F)). */
uint64_t crk_wire_size_d2h(uint64_t bytes, int32_t cuda_err, uint32_t frag_payload);
/* Encodes REPLY(xid, SUCCESS) | int err | [err == 0: opaque data<> = src[0..bytes)], framed with
 * cfg.frag_payload, into ring `out` at cursor out_off.  *wire_bytes (host) = its size, synchronously. */
int crk_xdr_encode_memcpy_d2h(crk_ctx* ctx, uint32_t xid, const void* src, uint64_t bytes, int32_t cuda_err,
                              crk_ring out, uint64_t out_off, uint64_t* wire_bytes, crk_stream_t stream);
/* n replies back to back from out_off in request order; arrays are dev arrays of length n.
 * wire_offs (dev, n entries) receives each reply's cursor, total_dev the sum of wire sizes. */
int crk_xdr_encode_memcpy_d2h_batch(crk_ctx* ctx, uint32_t n, const uint32_t* xids, const void* const* srcs,
                                    const uint64_t* bytes, const int32_t* cuda_errs, crk_ring out, uint64_t out_off,
                                    uint64_t* wire_offs, uint64_t* total_dev, crk_stream_t stream);
/* Generic batched REPLY encoder (control-path results): request i becomes
 *   REPLY(xid, MSG_ACCEPTED, AUTH_NONE, SUCCESS) | int err | [err == 0 && kind != 0: one XDR item]
 * where the item is `value` for CRK_K_U32 / CRK_K_U64, or `count` elements (bytes for opaque kinds)
 * read from device memory at `src` for the opaque / array kinds (VAR kinds carry their count word,
 * FIX kinds do not).  Replies are framed with cfg.frag_payload and written back to back from out_off
 * in request order; wire_offs (dev, n) receives each reply's cursor, total_dev the sum.  reqs_dev is a
 * device array owned by the caller; a kind outside 1..16 encodes no item (as kind 0); a request
 * with err == 0 whose item cannot be encoded (count >= 2^32, count > 0 with src NULL, src not
 * aligned to the element size) is encoded with err = CRK_E_ARG and no item.  Returns
 * CRK_E_ARG for n > cfg.max_jobs or a bad ring, CRK_E_CUDA on launch failure. */
typedef struct {
  uint32_t xid;
  int32_t err;
  uint32_t kind;
  uint32_t pad_;
  uint64_t value;
  const void* src;
  uint64_t count;
} crk_reply_req;
int crk_rpc_encode_replies_batch(crk_ctx* ctx, uint32_t n, const crk_reply_req* reqs_dev, crk_ring out,
                                 uint64_t out_off, uint64_t* wire_offs, uint64_t* total_dev, crk_stream_t stream);
/* REPLY | int err | [err == 0: T data<> big-endian] (typed analogue of the memcpy reply). */
int crk_xdr_encode_array_i32(crk_ctx*, uint32_t xid, const int32_t* src, uint64_t count, int32_t err, crk_ring out,
                             uint64_t out_off, uint64_t* wire_bytes, crk_stream_t);
int crk_xdr_encode_array_u32(crk_ctx*, uint32_t xid, const uint32_t* src, uint64_t count, int32_t err, crk_ring out,
                             uint64_t out_off, uint64_t* wire_bytes, crk_stream_t);
int crk_xdr_encode_array_i64(crk_ctx*, uint32_t xid, const int64_t* src, uint64_t count, int32_t err, crk_ring out,
                             uint64_t out_off, uint64_t* wire_bytes, crk_stream_t);
int crk_xdr_encode_array_u64(crk_ctx*, uint32_t xid, const uint64_t* src, uint64_t count, int32_t err, crk_ring out,
                             uint64_t out_off, uint64_t* wire_bytes, crk_stream_t);
int crk_xdr_encode_array_f32(crk_ctx*, uint32_t xid, const float* src, uint64_t count, int32_t err, crk_ring out,
                             uint64_t out_off, uint64_t* wire_bytes, crk_stream_t);
int crk_xdr_encode_array_f64(crk_ctx*, uint32_t xid, const double* src, uint64_t count, int32_t err, crk_ring out,
                             uint64_t out_off, uint64_t* wire_bytes, crk_stream_t);

/* Client-side CALL encoder (the inverse of K1-K5; used to fill rings and for round trips):
 * CALL header (AUTH_NONE cred/verf) for cfg.prog/vers and `proc`, then items in order.  For U32/U64
 * items `value` is the scalar; for the others `src` (device) holds count elements in host order.
 * Framing: greedy with cfg.frag_payload, or, if frag_lens (host array) is given, exactly those
 * fragment lengths (they must sum to the logical size; zero lengths allowed).  *wire_bytes (host) is
 * set synchronously. */
typedef struct {
  uint32_t kind, pad_;
  uint64_t value;    /* U32 / U64 */
  const void* src;   /* device pointer for opaque / array kinds */
  uint64_t count;    /* bytes (opaque) or elements (arrays) */
} crk_item_src;
int crk_rpc_encode_call(crk_ctx* ctx, uint32_t xid, uint32_t proc, const crk_item_src* items, uint32_t n_items,
                        const uint32_t* frag_lens, uint32_t n_lens, crk_ring out, uint64_t out_off,
                        uint64_t* wire_bytes, crk_stream_t stream);
/* Logical (unframed) size of such a CALL; pure host helper. */
uint64_t crk_call_logical_size(const crk_item_src* items, uint32_t n_items);

/* ---------------------------------------------------------------- the server step
 * One pass of the whole path over n_rings client streams (the north-star loop):
 * scan + parse every ring window, then for each record in index order
 *   wire error -> no reply; later duplicate xid -> E_XID, no reply;
 *   proc_h2d: E_SIZE / E_PTR (ptr range outside [region_base, +region_bytes)) -> reply err = 1,
 *             else copy the payload to ptr and reply err = 0;
 *   proc_d2h: E_PTR -> reply err = 1 (void arm), else reply err = 0 + the `size` bytes at ptr;
 *   proc_h2d_stripe: E_SIZE (strict n != size; offset + n > total) / E_PTR (ptr + offset range outside the
 *             region) -> no reply; else the bytes land at ptr + offset and, when the step holds every stripe of
 *             the memcpy (over all rings: sizes sum to total, ptr and total agree, one stripe at offset 0), the
 *             offset-0 stripe's place in its ring gets the memcpy's reply REPLY(parent) | int 0 (reading R22);
 *   other registered procs -> OK, no reply (decode them per argument).
 * Replies of ring r are framed with cfg.frag_payload and appended to send_rings[r] from cursor
 * send_offs[r] in record order.  All HtoD destinations and DtoH sources of one call must be disjoint
 * (the batch runs concurrently; reading R18).  Per-record results: crk_index_view serve_*;
 * per-ring: crk_index_ring_results. */
int crk_serve(crk_ctx* ctx, crk_index* idx, uint32_t n_rings, const crk_ring* rings, const uint64_t* heads,
              const uint64_t* tails, const crk_ring* send_rings, const uint64_t* send_offs, uint64_t region_base,
              uint64_t region_bytes, crk_stream_t stream);

/* A server step captured once as a CUDA graph and replayed as the rings advance (the server loop).
 * The ring cursors are read by the kernels at execution time from `doorbell` (device or mapped pinned
 * memory, uint64 [heads 0..n-1 | tails 0..n-1 | send_offs 0..n-1]), so a replay serves whatever
 * windows the host has published there; a ring whose published window is invalid (tail < head or
 * longer than its capacity) gets status CRK_E_ARG and no records.  Everything else (rings, send rings,
 * region, index, context) is fixed at capture.  The graph owns no memory of its own. */
typedef struct crk_graph crk_graph;
int crk_serve_graph_create(crk_ctx* ctx, crk_index* idx, uint32_t n_rings, const crk_ring* rings,
                           const crk_ring* send_rings, uint64_t region_base, uint64_t region_bytes,
                           const uint64_t* doorbell, crk_graph** out);
int crk_graph_launch(crk_graph* graph, crk_stream_t stream);
void crk_graph_destroy(crk_graph* graph);

/* ---------------------------------------------------------------- persistent server
 * The API-latency side of the paper: Cricket's overhead tracks the number of forwarded calls, most of them
 * small (Fig. 6 at P:228-234).  crk_server_start launches ONE resident CTA on `stream` that
 * polls a doorbell and runs every published step in place -- the crk_serve semantics above (scan, parse,
 * per-record decisions, HtoD copies, framed replies), with the same index tables and per-ring results --
 * with no kernel launch per step.  It is meant for streams of small calls (control RPCs, small memcpys):
 * one CTA moves the payloads, so bulk batches belong to crk_serve.
 *
 * Protocol.  The bell is caller-owned memory the device can read and write (mapped pinned host memory from
 * crk_host_alloc, or device memory).  To run a step the host writes head/tail/send_off for every ring,
 * then increments `seq` (a plain store after the others; x86 stores are ordered).  The kernel sees the new
 * seq (system-scope acquire), serves the windows, copies the per-ring results into `res`, sets `status`
 * and the device-timer stamps, and publishes done_seq = seq (system-scope release).  A window with
 * tail < head or longer than its ring is served as an empty ring with status CRK_E_ARG.  Setting `stop`
 * (then bumping seq) ends the kernel.  One step at a time: the host waits for done_seq == seq before
 * writing the next.
 *
 * Ownership.  While the server runs, it owns `ctx`'s scratch and `idx`: issue no other crk call on them
 * (other contexts are unaffected).  The kernel runs until stopped, so any host call that waits for the
 * whole device (cudaDeviceSynchronize, and allocator calls that synchronise implicitly) blocks until
 * crk_server_stop; use stream-ordered work on other non-blocking streams meanwhile.
 * The index must have max_records <= 1024 and 2 * max_records <=
 * the context's max_jobs.  crk_server_stop sets stop, waits for the kernel to exit and frees the handle
 * (not the bell). */
typedef struct {
  volatile uint64_t seq;       /* host -> device: step number (increment to run a step) */
  volatile uint64_t stop;      /* host -> device: nonzero ends the kernel at the next seq change */
  uint64_t head[CRK_MAX_RINGS];
  uint64_t tail[CRK_MAX_RINGS];
  uint64_t send_off[CRK_MAX_RINGS];
  volatile uint64_t done_seq;  /* device -> host: last completed step */
  volatile int32_t status;     /* device -> host: CRK_OK, or CRK_E_ARG when the step had an invalid window */
  uint32_t pad_;
  volatile uint64_t t_begin_ns, t_end_ns; /* device %globaltimer at the step's start (seq seen) and end */
  volatile uint64_t t_phase_ns[5];        /* device %globaltimer at the end of the step's setup, scan, parse,
                                             planning and mover phases */
  crk_ring_result res[CRK_MAX_RINGS];     /* device -> host: per-ring results of the last step */
} crk_server_bell;
typedef struct crk_server crk_server;
int crk_server_start(crk_ctx* ctx, crk_index* idx, uint32_t n_rings, const crk_ring* rings,
                     const crk_ring* send_rings, uint64_t region_base, uint64_t region_bytes, crk_server_bell* bell,
                     crk_stream_t stream, crk_server** out);
int crk_server_stop(crk_server* server);
/* One step through a running server whose bell is host memory (the protocol above, done in C so no
 * interpreter sits in the round trip): writes head/tail/send_off of the server's n_rings rings, bumps seq and
 * spins until done_seq == seq or timeout_ns elapses.  Returns the bell's status (CRK_OK, or CRK_E_ARG for an
 * invalid window); the per-ring results and device stamps are in the bell.  CRK_E_ARG also for a device-memory
 * bell or null arrays; CRK_E_CUDA when the step did not finish in time (the kernel failed or the timeout is too
 * short: the server is then in an unknown state -- stop it). */
int crk_server_step(crk_server* server, const uint64_t* heads, const uint64_t* tails, const uint64_t* send_offs,
                    uint64_t timeout_ns);

/* ---------------------------------------------------------------- memory utilities
 * Pinned, mapped, portable host memory for rings (cudaHostAlloc; with UVA the returned pointer is
 * also the device address), and a synchronous device->host copy for inspecting index tables. */
int crk_host_alloc(uint64_t bytes, void** out);
void crk_host_free(void* p);
int crk_copy_to_host(void* host_dst, const void* dev_src, uint64_t bytes);

/* ---------------------------------------------------------------- profiling
 * When enabled, CUDA events are recorded on the launching stream around each pipeline stage:
 * 0 = frame scan (K1; or the fused small-step front end, which also parses and plans), 1 = CALL parse (K3),
 * 2 = serve planning (statuses, K2 reply offsets, jobs),
 * 3 = the bulk mover (K4-K7).  crk_profile_read waits for the events, returns the summed device time
 * (ms[4]) and the number of timed launches (launches[4]) since the last read, and resets them. */
int crk_profile_enable(int on);
int crk_profile_read(double* ms, uint32_t* launches);

/* ---------------------------------------------------------------- misc */
const char* crk_strerror(int status);
int crk_last_cuda_error(void);   /* cudaError_t of the last CRK_E_CUDA */
int crk_kernel_launches(void);   /* number of kernels this process has launched through the library */
const char* crk_version(void);

#ifdef __cplusplus
}
#endif
#endif /* CRK_H */
