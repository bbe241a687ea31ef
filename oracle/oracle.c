/*
 * ORACLE — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, byte-at-a-time CPU implementation of what the crk hot path computes:
 * ONC RPC record marking (RFC 5531 §11), the RPC CALL/REPLY headers (RFC 5531 §8.2, §9) and the XDR
 * encodings of the memcpy arguments and typed arrays (RFC 4506 §3, §4.1-4.13).  The paper names
 * RFC 5531 as the RPC protocol (§3.4; ref [22] PAPER.md:285) and requires fragmented
 * messages for large parameters (§2); the server path it describes is "Cricket receives
 * the data in a buffer and transfers it to the GPU" (§4.2).  The byte-level rules come
 * from the RFCs; every reading of a point the paper is silent on is listed in DESIGN.md §3.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may load
 * this library.  It shares no code, header or constant with the CUDA path (include/crk.h,
 * paper_conf_sc_eilingkkflm23_b200/csrc): the status numbers below are restated from DESIGN.md §4.
 * Nothing here is tuned; it is written to be checked against the RFC text by eye.
 *
 * Pins (tests/test_oracle_*.py): RFC 4506 §7 worked example, glibc's Sun-RPC XDR (xdr_callmsg,
 * xdr_replymsg, xdrrec_*, xdr_u_hyper, xdr_bytes, xdr_float, xdr_double) called via dlvsym, Python
 * xdrlib, numpy big-endian views, brute force over every fragment split of tiny records, closed forms.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ---- status codes ---- */
#define OR_OK 0
#define OR_INCOMPLETE 1
#define OR_E_ARG (-1)
#define OR_E_TRUNCATED (-2)
#define OR_E_FRAG (-3)
#define OR_E_RPC (-4)
#define OR_E_AUTH (-5)
#define OR_E_PAD (-6)
#define OR_E_SIZE (-7)
#define OR_E_TRAILING (-8)
#define OR_E_XID (-9)
#define OR_E_PTR (-10)
#define OR_E_CAPACITY (-11)
#define OR_E_PROC (-12)

/* ---- XDR item kinds of a procedure's argument schema ---- */
#define OR_K_U32 1        /* unsigned int / int / enum / bool: 4 bytes, RFC 4506 §4.1-4.4 */
#define OR_K_U64 2        /* unsigned hyper / hyper: 8 bytes, RFC 4506 §4.5 */
#define OR_K_OPAQUE_VAR 3 /* opaque<>: length word + bytes + zero pad, RFC 4506 §4.10 (string §4.11 too) */
#define OR_K_OPAQUE_FIX 4 /* opaque[n]: bytes + zero pad, RFC 4506 §4.9 */
#define OR_K_I32_VAR 5    /* int<>, RFC 4506 §4.13 */
#define OR_K_U32_VAR 6
#define OR_K_F32_VAR 7    /* float<>: IEEE single, RFC 4506 §4.6 */
#define OR_K_I64_VAR 8    /* hyper<> */
#define OR_K_U64_VAR 9
#define OR_K_F64_VAR 10   /* double<>: IEEE double, RFC 4506 §4.7 */
#define OR_K_I32_FIX 11   /* int[n], RFC 4506 §4.12 */
#define OR_K_U32_FIX 12
#define OR_K_F32_FIX 13
#define OR_K_I64_FIX 14
#define OR_K_U64_FIX 15
#define OR_K_F64_FIX 16

#define OR_AUTH_MAX 400u  /* RFC 5531 §8.2: opaque body<400> */
#define OR_MAX_ITEMS 8

/* element size in bytes of an array kind (1 for opaque), 0 for a scalar kind */
static uint32_t or_elem_size(uint32_t kind) {
  switch (kind) {
    case OR_K_OPAQUE_VAR: case OR_K_OPAQUE_FIX: return 1;
    case OR_K_I32_VAR: case OR_K_U32_VAR: case OR_K_F32_VAR:
    case OR_K_I32_FIX: case OR_K_U32_FIX: case OR_K_F32_FIX: return 4;
    case OR_K_I64_VAR: case OR_K_U64_VAR: case OR_K_F64_VAR:
    case OR_K_I64_FIX: case OR_K_U64_FIX: case OR_K_F64_FIX: return 8;
    default: return 0;
  }
}
static int or_kind_is_var(uint32_t kind) {
  return kind == OR_K_OPAQUE_VAR || (kind >= OR_K_I32_VAR && kind <= OR_K_F64_VAR);
}

/* RFC 4506 §3: every item is padded to a multiple of four bytes with zero bytes. */
static uint64_t or_pad(uint64_t n) { return (4 - (n % 4)) % 4; }

/* RFC 4506 §4.1: big-endian: byte 0 is the most significant. */
uint32_t or_be32(const uint8_t* b) {
  return ((uint32_t)b[0] << 24) | ((uint32_t)b[1] << 16) | ((uint32_t)b[2] << 8) | (uint32_t)b[3];
}
static void or_put_be32(uint8_t* b, uint32_t v) {
  b[0] = (uint8_t)(v >> 24); b[1] = (uint8_t)(v >> 16); b[2] = (uint8_t)(v >> 8); b[3] = (uint8_t)v;
}

/* =====================================================================================
 * XDR encoding primitives, each appending to out at *pos and returning the new position.
 * ===================================================================================== */

/* RFC 4506 §4.1/§4.2: 4-byte big-endian integer. */
uint64_t or_xdr_put_u32(uint8_t* out, uint64_t pos, uint32_t v) {
  or_put_be32(out + pos, v);
  return pos + 4;
}
/* RFC 4506 §4.5: hyper is 8 bytes, most significant word first ("bytes 0..7, byte 0 MSB"). */
uint64_t or_xdr_put_u64(uint8_t* out, uint64_t pos, uint64_t v) {
  pos = or_xdr_put_u32(out, pos, (uint32_t)(v >> 32));
  return or_xdr_put_u32(out, pos, (uint32_t)(v & 0xffffffffu));
}
/* RFC 4506 §4.9: fixed-length opaque: n bytes then (-n mod 4) zero bytes. */
uint64_t or_xdr_put_opaque_fix(uint8_t* out, uint64_t pos, const uint8_t* data, uint64_t n) {
  uint64_t i;
  for (i = 0; i < n; ++i) out[pos + i] = data[i];
  for (i = 0; i < or_pad(n); ++i) out[pos + n + i] = 0;
  return pos + n + or_pad(n);
}
/* RFC 4506 §4.10: variable-length opaque: unsigned length n, then as §4.9. */
uint64_t or_xdr_put_opaque_var(uint8_t* out, uint64_t pos, const uint8_t* data, uint32_t n) {
  pos = or_xdr_put_u32(out, pos, n);
  return or_xdr_put_opaque_fix(out, pos, data, n);
}
/* RFC 4506 §4.12 (fixed array) / §4.13 (counted array) of 4- or 8-byte elements.
 * `elems` holds count elements in host (little-endian) byte order; each is written big-endian. */
uint64_t or_xdr_put_array(uint8_t* out, uint64_t pos, const uint8_t* elems, uint32_t count, uint32_t esize,
                          int with_count) {
  uint64_t i;
  uint32_t j;
  if (with_count) pos = or_xdr_put_u32(out, pos, count);
  for (i = 0; i < count; ++i)
    for (j = 0; j < esize; ++j) out[pos + i * esize + j] = elems[i * esize + (esize - 1 - j)];
  return pos + (uint64_t)count * esize;
}

/* RFC 5531 §9 (struct rpc_msg / call_body) with AUTH_NONE-style opaque_auth (§8.2) cred and verf. */
uint64_t or_rpc_put_call_header(uint8_t* out, uint64_t pos, uint32_t xid, uint32_t prog, uint32_t vers,
                                uint32_t proc, uint32_t cred_flavor, const uint8_t* cred, uint32_t cred_len,
                                uint32_t verf_flavor, const uint8_t* verf, uint32_t verf_len) {
  pos = or_xdr_put_u32(out, pos, xid);
  pos = or_xdr_put_u32(out, pos, 0); /* msg_type CALL = 0 */
  pos = or_xdr_put_u32(out, pos, 2); /* rpcvers = 2 */
  pos = or_xdr_put_u32(out, pos, prog);
  pos = or_xdr_put_u32(out, pos, vers);
  pos = or_xdr_put_u32(out, pos, proc);
  pos = or_xdr_put_u32(out, pos, cred_flavor);
  pos = or_xdr_put_opaque_var(out, pos, cred, cred_len);
  pos = or_xdr_put_u32(out, pos, verf_flavor);
  pos = or_xdr_put_opaque_var(out, pos, verf, verf_len);
  return pos;
}
/* RFC 5531 §9: REPLY, MSG_ACCEPTED, verf AUTH_NONE (flavor 0, empty body), accept_stat SUCCESS. */
uint64_t or_rpc_put_reply_header(uint8_t* out, uint64_t pos, uint32_t xid) {
  pos = or_xdr_put_u32(out, pos, xid);
  pos = or_xdr_put_u32(out, pos, 1); /* msg_type REPLY */
  pos = or_xdr_put_u32(out, pos, 0); /* reply_stat MSG_ACCEPTED */
  pos = or_xdr_put_u32(out, pos, 0); /* verf flavor AUTH_NONE */
  pos = or_xdr_put_u32(out, pos, 0); /* verf body length 0 */
  pos = or_xdr_put_u32(out, pos, 0); /* accept_stat SUCCESS */
  return pos;
}

/* =====================================================================================
 * Record marking (RFC 5531 §11).
 * A record is one or more fragments; each fragment is a 4-byte header (bit 31: last fragment,
 * bits 0-30: length) followed by that many bytes.
 * ===================================================================================== */

/* Number of fragments greedy framing with payload F gives a record of n logical bytes:
 * the first k-1 carry exactly F bytes, the last the remainder, and there is always >= 1 fragment
 * (reading R3: no empty trailing fragment when F divides n). */
uint64_t or_frame_count(uint64_t n, uint32_t F) {
  if (n == 0) return 1;
  return (n + F - 1) / F;
}
uint64_t or_frame_wire_size(uint64_t n, uint32_t F) { return n + 4 * or_frame_count(n, F); }

/* Greedy framing: writes the wire record for logical bytes L[0..n) and returns its size. */
uint64_t or_frame_record(const uint8_t* L, uint64_t n, uint32_t F, uint8_t* out) {
  uint64_t k = or_frame_count(n, F), pos = 0, f, i;
  for (f = 0; f < k; ++f) {
    uint64_t len = (f + 1 < k) ? F : n - (k - 1) * (uint64_t)F;
    uint32_t h = (uint32_t)len | ((f + 1 == k) ? 0x80000000u : 0u);
    or_put_be32(out + pos, h);
    pos += 4;
    for (i = 0; i < len; ++i) out[pos + i] = L[f * (uint64_t)F + i];
    pos += len;
  }
  return pos;
}
/* Framing with an explicit list of fragment lengths (lens[0..k), summing to n; the last one carries
 * the last-fragment bit).  Zero lengths are allowed (RFC 5531 §11 permits 0 .. 2^31-1). */
uint64_t or_frame_record_lens(const uint8_t* L, uint64_t n, const uint32_t* lens, uint64_t k, uint8_t* out) {
  uint64_t pos = 0, lpos = 0, f, i;
  for (f = 0; f < k; ++f) {
    uint32_t h = lens[f] | ((f + 1 == k) ? 0x80000000u : 0u);
    or_put_be32(out + pos, h);
    pos += 4;
    for (i = 0; i < lens[f]; ++i) out[pos + i] = L[lpos + i];
    pos += lens[f];
    lpos += lens[f];
  }
  (void)n;
  return pos;
}

typedef struct {
  uint64_t phys;   /* ring cursor of the fragment's first data byte (header position + 4) */
  uint64_t lstart; /* logical offset of that byte within its record */
  uint32_t len;    /* fragment data length */
  uint32_t last;   /* 1 on the record's final fragment */
  uint32_t rec;    /* record number within this scan */
  uint32_t pad_;
} or_frag;

typedef struct {
  uint64_t begin;  /* ring cursor of the first header */
  uint64_t end;    /* ring cursor one past the last data byte */
  uint64_t len;    /* logical length = sum of fragment lengths */
  uint32_t frag0;  /* index of the first fragment */
  uint32_t nfrags;
} or_rec;

static uint8_t or_ring_at(const uint8_t* ring, uint64_t cap, uint64_t pos) { return ring[pos & (cap - 1)]; }

/* Frame decode (RFC 5531 §11) over the ring window [head, tail) (cursors; byte at ring[c & (cap-1)]).
 * Checks for each header at cursor p, in this order (reading R1/R2/R8):
 *   1. fewer than 4 bytes left           -> stop: OK if p == r0 == tail, else INCOMPLETE
 *   2. sum + len > max_record_bytes       -> E_FRAG
 *   3. p + 4 + len > tail                 -> INCOMPLETE
 *   4. index full (frags, or records at a record's first fragment)
 *                                         -> INCOMPLETE if >= 1 record was emitted, else E_CAPACITY
 * In every stop case consumed = r0 (start of the record being built) and its fragments are dropped. */
int or_frame_scan(const uint8_t* ring, uint64_t cap, uint64_t head, uint64_t tail, uint64_t max_record_bytes,
                  uint32_t max_frags, uint32_t max_records, or_frag* frags, uint32_t* n_frags, or_rec* recs,
                  uint32_t* n_recs, uint64_t* consumed) {
  uint64_t p = head, r0 = head, sum = 0;
  uint32_t nf = 0, nr = 0, f0 = 0;
  int st;
  if (cap == 0 || (cap & (cap - 1)) != 0 || tail < head || tail - head > cap) return OR_E_ARG;
  for (;;) {
    uint32_t h, len, last;
    if (tail - p < 4) { st = (p == r0 && p == tail) ? OR_OK : OR_INCOMPLETE; break; }
    h = ((uint32_t)or_ring_at(ring, cap, p) << 24) | ((uint32_t)or_ring_at(ring, cap, p + 1) << 16) |
        ((uint32_t)or_ring_at(ring, cap, p + 2) << 8) | (uint32_t)or_ring_at(ring, cap, p + 3);
    last = h >> 31;
    len = h & 0x7fffffffu;
    if (sum + len > max_record_bytes) { st = OR_E_FRAG; break; }
    if (p + 4 + (uint64_t)len > tail) { st = OR_INCOMPLETE; break; }
    if (nf == max_frags || (p == r0 && nr == max_records)) { st = nr > 0 ? OR_INCOMPLETE : OR_E_CAPACITY; break; }
    frags[nf].phys = p + 4;
    frags[nf].lstart = sum;
    frags[nf].len = len;
    frags[nf].last = last;
    frags[nf].rec = nr;
    frags[nf].pad_ = 0;
    nf++;
    sum += len;
    p += 4 + (uint64_t)len;
    if (last) {
      recs[nr].begin = r0;
      recs[nr].end = p;
      recs[nr].len = sum;
      recs[nr].frag0 = f0;
      recs[nr].nfrags = nf - f0;
      nr++;
      r0 = p;
      f0 = nf;
      sum = 0;
    }
  }
  *n_frags = f0; /* fragments of the unfinished record are dropped */
  *n_recs = nr;
  *consumed = r0;
  return st;
}

/* Logical record: the concatenation of its fragments' data (RFC 5531 §11). */
void or_record_logical(const uint8_t* ring, uint64_t cap, const or_frag* frags, const or_rec* rec, uint8_t* L) {
  uint64_t o = 0, i;
  uint32_t f;
  for (f = rec->frag0; f < rec->frag0 + rec->nfrags; ++f)
    for (i = 0; i < frags[f].len; ++i) L[o++] = or_ring_at(ring, cap, frags[f].phys + i);
}

/* =====================================================================================
 * CALL parse (RFC 5531 §9, §8.2) and arguments by schema (RFC 4506).
 * ===================================================================================== */

typedef struct {
  uint32_t proc;
  uint32_t n_items;
  uint32_t items[OR_MAX_ITEMS]; /* kind | (fixed count << 8) */
} or_schema;

typedef struct {
  uint32_t prog, vers;
  int strict;            /* 1: nonzero pad -> E_PAD, unconsumed bytes -> E_TRAILING, opaque n != size -> E_SIZE */
  uint32_t proc_h2d;     /* built-in (ptr u64, mem opaque<>, size u64) */
  uint32_t proc_d2h;     /* built-in (ptr u64, size u64) */
  uint32_t proc_stripe;  /* built-in (ptr u64, mem opaque<>, size u64, parent u32, offset u64, total u64); 0: off */
} or_cfg;

typedef struct {
  int32_t status;        /* first wire-level failure, or OK */
  uint32_t xid, proc, n_items;
  uint32_t kind[OR_MAX_ITEMS];
  uint64_t off[OR_MAX_ITEMS];   /* logical offset of the item's data (after its count word, if any) */
  uint64_t count[OR_MAX_ITEMS]; /* opaque: bytes; arrays: elements; scalars: 0 */
  uint64_t value[OR_MAX_ITEMS]; /* scalars: the decoded value */
  uint64_t end;          /* logical offset after the last argument */
} or_call;

static int or_get_u32(const uint8_t* L, uint64_t n, uint64_t* o, uint32_t* v) {
  if (*o + 4 > n) return OR_E_TRUNCATED;
  *v = or_be32(L + *o);
  *o += 4;
  return OR_OK;
}

/* Reads opaque_auth (RFC 5531 §8.2): flavor, body<400>. */
static int or_get_auth(const uint8_t* L, uint64_t n, uint64_t* o, int strict) {
  uint32_t flavor, len;
  uint64_t i;
  int st;
  if ((st = or_get_u32(L, n, o, &flavor))) return st;
  if ((st = or_get_u32(L, n, o, &len))) return st;
  if (len > OR_AUTH_MAX) return OR_E_AUTH;
  if (*o + len + or_pad(len) > n) return OR_E_TRUNCATED;
  if (strict)
    for (i = 0; i < or_pad(len); ++i)
      if (L[*o + len + i] != 0) return OR_E_PAD;
  *o += len + or_pad(len);
  return OR_OK;
}

static const or_schema* or_find_schema(const or_schema* schemas, uint32_t n_schemas, uint32_t proc) {
  uint32_t i;
  for (i = 0; i < n_schemas; ++i)
    if (schemas[i].proc == proc) return &schemas[i];
  return 0;
}

/* Parses the logical record L[0..n) as a CALL.  Checks run in logical-offset order; the first failure
 * is the record's status (DESIGN.md §4 "error precedence"). */
int or_parse_call(const uint8_t* L, uint64_t n, const or_cfg* cfg, const or_schema* schemas, uint32_t n_schemas,
                  or_call* c) {
  uint64_t o = 0, i;
  uint32_t v, it;
  int st;
  const or_schema* sc;
  memset(c, 0, sizeof(*c));
#define OR_FAIL(s) do { c->status = (s); c->end = o; return c->status; } while (0)
  if ((st = or_get_u32(L, n, &o, &c->xid))) OR_FAIL(st);
  if ((st = or_get_u32(L, n, &o, &v))) OR_FAIL(st);
  if (v != 0) OR_FAIL(OR_E_RPC);                 /* msg_type must be CALL */
  if ((st = or_get_u32(L, n, &o, &v))) OR_FAIL(st);
  if (v != 2) OR_FAIL(OR_E_RPC);                 /* rpcvers must be 2 */
  if ((st = or_get_u32(L, n, &o, &v))) OR_FAIL(st);
  if (v != cfg->prog) OR_FAIL(OR_E_RPC);
  if ((st = or_get_u32(L, n, &o, &v))) OR_FAIL(st);
  if (v != cfg->vers) OR_FAIL(OR_E_RPC);
  if ((st = or_get_u32(L, n, &o, &c->proc))) OR_FAIL(st);
  sc = or_find_schema(schemas, n_schemas, c->proc);
  if (!sc) OR_FAIL(OR_E_PROC);
  if ((st = or_get_auth(L, n, &o, cfg->strict))) OR_FAIL(st); /* cred */
  if ((st = or_get_auth(L, n, &o, cfg->strict))) OR_FAIL(st); /* verf */
  c->n_items = sc->n_items;
  for (it = 0; it < sc->n_items; ++it) {
    uint32_t kind = sc->items[it] & 0xff, fixed = sc->items[it] >> 8, es = or_elem_size(kind);
    c->kind[it] = kind;
    if (kind == OR_K_U32) {
      if ((st = or_get_u32(L, n, &o, &v))) OR_FAIL(st);
      c->off[it] = o - 4;
      c->value[it] = v;
    } else if (kind == OR_K_U64) {
      uint32_t hi, lo;
      if ((st = or_get_u32(L, n, &o, &hi))) OR_FAIL(st);
      if ((st = or_get_u32(L, n, &o, &lo))) OR_FAIL(st);
      c->off[it] = o - 8;
      c->value[it] = ((uint64_t)hi << 32) | lo;
    } else {
      uint64_t cnt, bytes, padn;
      if (or_kind_is_var(kind)) {
        if ((st = or_get_u32(L, n, &o, &v))) OR_FAIL(st);
        cnt = v;
      } else {
        cnt = fixed;
      }
      bytes = cnt * es;
      padn = or_pad(bytes);   /* zero for 4/8-byte elements */
      if (o + bytes + padn > n) OR_FAIL(OR_E_TRUNCATED);
      if (cfg->strict)
        for (i = 0; i < padn; ++i)
          if (L[o + bytes + i] != 0) { o += bytes; OR_FAIL(OR_E_PAD); }
      c->off[it] = o;
      c->count[it] = cnt;
      o += bytes + padn;
    }
  }
  c->end = o;
  if (cfg->strict && o != n) { c->status = OR_E_TRAILING; return c->status; }
  c->status = OR_OK;
  return OR_OK;
#undef OR_FAIL
}

/* The built-in memcpy schemas (readings R9, R22; Cricket's RPCL is not in the paper): HtoD, DtoH and
 * the HtoD stripe (one part of a memcpy sent over one of several connections).  With
 * proc_stripe == 0 the third entry repeats the HtoD schema (the first match wins, so it is never used). */
void or_builtin_schemas(const or_cfg* cfg, or_schema* out3) {
  memset(out3, 0, 3 * sizeof(or_schema));
  out3[0].proc = cfg->proc_h2d;
  out3[0].n_items = 3;
  out3[0].items[0] = OR_K_U64;
  out3[0].items[1] = OR_K_OPAQUE_VAR;
  out3[0].items[2] = OR_K_U64;
  out3[1].proc = cfg->proc_d2h;
  out3[1].n_items = 2;
  out3[1].items[0] = OR_K_U64;
  out3[1].items[1] = OR_K_U64;
  if (cfg->proc_stripe == 0) { out3[2] = out3[0]; return; }
  out3[2].proc = cfg->proc_stripe;
  out3[2].n_items = 6;
  out3[2].items[0] = OR_K_U64;        /* ptr: the destination of the whole memcpy */
  out3[2].items[1] = OR_K_OPAQUE_VAR; /* mem: this stripe's bytes */
  out3[2].items[2] = OR_K_U64;        /* size */
  out3[2].items[3] = OR_K_U32;        /* parent: the memcpy's xid */
  out3[2].items[4] = OR_K_U64;        /* offset of this stripe within the memcpy */
  out3[2].items[5] = OR_K_U64;        /* total bytes of the memcpy */
}

/* =====================================================================================
 * Decode of one parsed CALL into caller memory.
 * ===================================================================================== */

/* memcpy HtoD: dst[0..m) = the opaque payload, nothing else written.
 * Order: wire status, proc, E_SIZE (strict: n == size), E_PTR (dst too small). */
int or_decode_memcpy_h2d(const uint8_t* L, const or_call* c, const or_cfg* cfg, uint8_t* dst, uint64_t dst_bytes,
                         uint64_t* copied) {
  uint64_t n, size, m, i;
  *copied = 0;
  if (c->status != OR_OK) return c->status;
  if (c->proc != cfg->proc_h2d) return OR_E_PROC;
  n = c->count[1];
  size = c->value[2];
  if (cfg->strict && n != size) return OR_E_SIZE;
  m = (cfg->strict || n <= size) ? n : size;
  if (dst_bytes < m) return OR_E_PTR;
  for (i = 0; i < m; ++i) dst[i] = L[c->off[1] + i];
  *copied = m;
  return OR_OK;
}

/* Typed array or opaque argument arg_no (RFC 4506 §4.9-4.13): element i is the big-endian bytes at
 * off + s*i, byte-reversed into host order.  Floats are moved as bit patterns (reading R13).
 * Order: wire status, E_ARG (arg is not of `kind`), E_SIZE (count > max_count). */
int or_decode_item(const uint8_t* L, const or_call* c, uint32_t arg_no, uint32_t kind, uint8_t* dst,
                   uint64_t max_count, uint64_t* count) {
  uint64_t i, cnt;
  uint32_t s, j;
  *count = 0;
  if (c->status != OR_OK) return c->status;
  if (arg_no >= c->n_items || c->kind[arg_no] != kind || or_elem_size(kind) == 0) return OR_E_ARG;
  cnt = c->count[arg_no];
  if (cnt > max_count) return OR_E_SIZE;
  s = or_elem_size(kind);
  for (i = 0; i < cnt; ++i)
    for (j = 0; j < s; ++j) dst[i * s + j] = L[c->off[arg_no] + i * s + (s - 1 - j)];
  *count = cnt;
  return OR_OK;
}

/* =====================================================================================
 * memcpy DtoH reply encode (RFC 5531 §9 + the mem_result union, reading R10):
 *   REPLY header (24 B) | int err | if err == 0: opaque data<> (length, bytes, zero pad)
 * framed greedily with payload F.  Returns the wire size; out may be NULL to only size it.
 * ===================================================================================== */
uint64_t or_reply_logical_size(uint64_t n, int32_t err) { return err == 0 ? 24 + 4 + 4 + n + or_pad(n) : 24 + 4; }

uint64_t or_encode_memcpy_d2h(uint32_t xid, const uint8_t* src, uint32_t n, int32_t err, uint32_t F, uint8_t* out) {
  uint64_t ln = or_reply_logical_size(n, err), pos = 0, w;
  uint8_t* L;
  if (!out) return or_frame_wire_size(ln, F);
  L = (uint8_t*)malloc(ln ? ln : 1);
  pos = or_rpc_put_reply_header(L, pos, xid);
  pos = or_xdr_put_u32(L, pos, (uint32_t)err);
  if (err == 0) pos = or_xdr_put_opaque_var(L, pos, src, n);
  w = or_frame_record(L, pos, F, out);
  free(L);
  return w;
}

/* Typed array reply: REPLY header | int err | if err == 0: T data<> (count, big-endian elements). */
uint64_t or_encode_array_reply(uint32_t xid, const uint8_t* elems, uint32_t count, uint32_t esize, int32_t err,
                               uint32_t F, uint8_t* out) {
  uint64_t ln = err == 0 ? 24 + 4 + 4 + (uint64_t)count * esize : 28, pos = 0, w;
  uint8_t* L;
  if (!out) return or_frame_wire_size(ln, F);
  L = (uint8_t*)malloc(ln);
  pos = or_rpc_put_reply_header(L, pos, xid);
  pos = or_xdr_put_u32(L, pos, (uint32_t)err);
  if (err == 0) pos = or_xdr_put_array(L, pos, elems, count, esize, 1);
  w = or_frame_record(L, pos, F, out);
  free(L);
  return w;
}

/* Generic REPLY (control-path results): REPLY header | int err | [err == 0 && kind != 0: one item]:
 * U32 / U64 -> value; opaque kinds -> count bytes of elems (VAR with its length word); array kinds ->
 * count elements of elems in host order written big-endian (VAR with its count word). */
uint64_t or_encode_reply_item(uint32_t xid, int32_t err, uint32_t kind, uint64_t value, const uint8_t* elems,
                              uint32_t count, uint32_t F, uint8_t* out) {
  uint64_t cap = 28 + 8 + (uint64_t)count * 8 + 8, pos = 0, w;
  uint8_t* L = (uint8_t*)malloc(cap);
  pos = or_rpc_put_reply_header(L, pos, xid);
  pos = or_xdr_put_u32(L, pos, (uint32_t)err);
  if (err == 0 && kind != 0) {
    if (kind == OR_K_U32) pos = or_xdr_put_u32(L, pos, (uint32_t)value);
    else if (kind == OR_K_U64) pos = or_xdr_put_u64(L, pos, value);
    else if (kind == OR_K_OPAQUE_VAR) pos = or_xdr_put_opaque_var(L, pos, elems, count);
    else if (kind == OR_K_OPAQUE_FIX) pos = or_xdr_put_opaque_fix(L, pos, elems, count);
    else pos = or_xdr_put_array(L, pos, elems, count, or_elem_size(kind), or_kind_is_var(kind));
  }
  if (!out) { free(L); return or_frame_wire_size(pos, F); }
  w = or_frame_record(L, pos, F, out);
  free(L);
  return w;
}

/* =====================================================================================
 * Server step over several rings (the north-star loop): frame-scan each ring, parse
 * every CALL, then in index order (ring 0's records first):
 *   - wire-level failure          -> status, no reply
 *   - xid seen earlier in index   -> E_XID, no reply (reading R11)
 *   - memcpy HtoD: E_SIZE / E_PTR (region) -> reply err=1; else copy to region at ptr, reply err=0
 *   - memcpy DtoH: E_PTR (region) -> reply err=1 (void arm); else reply err=0 + data from region at ptr
 *   - any other registered proc   -> OK, no reply (decoded per argument by the caller)
 * Replies of ring r are appended, framed with F, to send ring r from cursor out_off[r].
 * ===================================================================================== */
typedef struct {
  int32_t status;
  int32_t reply_err;  /* -1: no reply */
  uint32_t ring, xid, proc, pad_;
  uint64_t reply_off; /* send-ring cursor of the reply (if any) */
  uint64_t reply_wire;
} or_serve_rec;

/* memcpy HtoD stripe (reading R22; SURVEY.md §8(f) NEXT-1 -- Cricket's parallel-socket memcpy,
 * PAPER.md:170, :238, :240): a memcpy of `total` bytes to `ptr` sent as several CALLs, one per connection, each
 * carrying bytes [offset, offset + size) and the memcpy's own xid as `parent`.  Checks of one stripe, in order:
 * strict mem.n == size (E_SIZE); total < 2^63 and offset + m <= total (E_SIZE); [ptr + offset, + m) inside the
 * region (E_PTR).  A stripe that passes copies its bytes and has no reply of its own. */
static int or_stripe_check(const or_call* c, const or_cfg* cfg, uint64_t region_base, uint64_t region_bytes,
                           uint64_t* m_out) {
  uint64_t n = c->count[1], size = c->value[2], ptr = c->value[0], off = c->value[4], tot = c->value[5];
  uint64_t m = (cfg->strict || n <= size) ? n : size;
  *m_out = 0;
  if (cfg->strict && n != size) return OR_E_SIZE;
  if (tot >= (1ull << 63) || off > tot || m > tot - off) return OR_E_SIZE;
  if (ptr > ~0ull - off) return OR_E_PTR;
  ptr += off;
  if (ptr < region_base || m > region_bytes || ptr - region_base > region_bytes - m) return OR_E_PTR;
  *m_out = m;
  return OR_OK;
}

/* One parent memcpy of a serve step: it is complete when its OK stripes agree on (ptr, total), their sizes sum
 * to total, and one of them starts at offset 0 -- the lead, the earliest such stripe in index order, whose
 * record then carries the parent's reply REPLY(parent) | int 0 (the HtoD reply) in its ring's reply order. */
typedef struct {
  uint32_t parent, bad;
  uint64_t ptr, total, landed;
  uint32_t lead;         /* index of the lead record, or 0xffffffff */
  uint32_t nstripes;     /* OK stripes seen */
} or_parent;

static or_parent* or_parent_of(or_parent* ps, uint32_t* np, uint32_t parent) {
  uint32_t k;
  for (k = 0; k < *np; ++k)
    if (ps[k].parent == parent) return &ps[k];
  memset(&ps[*np], 0, sizeof(or_parent));
  ps[*np].parent = parent;
  ps[*np].lead = 0xffffffffu;
  return &ps[(*np)++];
}

int or_serve(uint32_t n_rings, const uint8_t* const* rings, const uint64_t* caps, const uint64_t* heads,
             const uint64_t* tails, uint64_t max_record_bytes, uint32_t max_frags_per_ring,
             uint32_t max_records_per_ring, const or_cfg* cfg, const or_schema* user_schemas, uint32_t n_user,
             uint8_t* region, uint64_t region_base, uint64_t region_bytes, uint8_t* const* send_rings,
             const uint64_t* send_caps, const uint64_t* out_off, uint32_t F, int32_t* scan_status,
             uint64_t* consumed, uint64_t* reply_bytes, or_serve_rec* out_recs, uint32_t max_out,
             uint32_t* n_out) {
  uint32_t r, i, total = 0, ns = n_user + 3, pass, n_parents = 0;
  or_schema* schemas = (or_schema*)calloc(ns, sizeof(or_schema));
  or_frag* frags = (or_frag*)malloc((size_t)(max_frags_per_ring ? max_frags_per_ring : 1) * sizeof(or_frag));
  or_rec* recs = (or_rec*)malloc((size_t)(max_records_per_ring ? max_records_per_ring : 1) * sizeof(or_rec));
  uint32_t* seen_xid = (uint32_t*)malloc((size_t)(max_out ? max_out : 1) * sizeof(uint32_t));
  uint8_t* xid_readable = (uint8_t*)malloc((size_t)(max_out ? max_out : 1));
  or_parent* parents = (or_parent*)malloc((size_t)(max_out ? max_out : 1) * sizeof(or_parent));
  or_builtin_schemas(cfg, schemas);
  for (i = 0; i < n_user; ++i) schemas[3 + i] = user_schemas[i];
  /* Pass 0 decides every record and gathers the stripes of each parent memcpy (a stripe's reply depends on
   * stripes in other rings); pass 1 repeats the same decisions and carries them out in index order. */
  for (pass = 0; pass < 2; ++pass) {
  total = 0;
  for (r = 0; r < n_rings; ++r) {
    uint32_t nf = 0, nr = 0;
    uint64_t w = out_off[r];
    scan_status[r] = or_frame_scan(rings[r], caps[r], heads[r], tails[r], max_record_bytes, max_frags_per_ring,
                                   max_records_per_ring, frags, &nf, recs, &nr, &consumed[r]);
    for (i = 0; i < nr; ++i) {
      or_call c;
      or_serve_rec* o;
      uint32_t j;
      int dup = 0;
      uint8_t* L = (uint8_t*)malloc(recs[i].len ? recs[i].len : 1);
      if (total >= max_out) { free(L); break; }
      or_record_logical(rings[r], caps[r], frags, &recs[i], L);
      or_parse_call(L, recs[i].len, cfg, schemas, ns, &c);
      o = &out_recs[total];
      memset(o, 0, sizeof(*o));
      o->ring = r;
      o->xid = c.xid;
      o->proc = c.proc;
      o->status = c.status;
      o->reply_err = -1;
      /* reading R11: the record owning an xid is the earliest one in index order whose xid word is
       * readable (logical length >= 4); a later record with the same xid is a duplicate. */
      for (j = 0; j < total; ++j)
        if (xid_readable[j] && seen_xid[j] == c.xid) dup = 1;
      seen_xid[total] = c.xid;
      xid_readable[total] = recs[i].len >= 4;
      if (o->status == OR_OK && dup) o->status = OR_E_XID;
      if (pass == 0) {  /* decisions only: gather the OK stripes of each parent */
        if (o->status == OR_OK && cfg->proc_stripe && c.proc == cfg->proc_stripe) {
          uint64_t m;
          if (or_stripe_check(&c, cfg, region_base, region_bytes, &m) == OR_OK) {
            or_parent* P = or_parent_of(parents, &n_parents, (uint32_t)c.value[3]);
            if (P->nstripes++ == 0) {  /* the first OK stripe fixes the memcpy's ptr and total */
              P->ptr = c.value[0];
              P->total = c.value[5];
            }
            if (P->ptr != c.value[0] || P->total != c.value[5]) P->bad = 1;
            P->landed += m;
            if (c.value[4] == 0 && P->lead == 0xffffffffu) P->lead = total;
          }
        }
        total++;
        free(L);
        continue;
      }
      if (o->status == OR_OK && cfg->proc_stripe && c.proc == cfg->proc_stripe) {
        uint64_t m, b;
        o->status = or_stripe_check(&c, cfg, region_base, region_bytes, &m);
        if (o->status == OR_OK) {
          const or_parent* P = or_parent_of(parents, &n_parents, (uint32_t)c.value[3]);
          uint64_t dst = c.value[0] + c.value[4] - region_base;
          for (b = 0; b < m; ++b) region[dst + b] = L[c.off[1] + b];
          if (P->lead == total && !P->bad && P->landed == P->total) {  /* the parent's reply */
            uint8_t tmp[32];
            uint64_t ln = or_rpc_put_reply_header(tmp, 0, P->parent), wl;
            ln = or_xdr_put_u32(tmp, ln, 0);
            wl = or_frame_wire_size(ln, F);
            if (send_rings) {
              uint8_t* wire = (uint8_t*)malloc(wl);
              or_frame_record(tmp, ln, F, wire);
              for (b = 0; b < wl; ++b) send_rings[r][(w + b) & (send_caps[r] - 1)] = wire[b];
              free(wire);
            }
            o->reply_err = 0;
            o->reply_off = w;
            o->reply_wire = wl;
            w += wl;
          }
        }
      } else if (o->status == OR_OK && c.proc == cfg->proc_h2d) {
        uint64_t n = c.count[1], size = c.value[2], ptr = c.value[0];
        uint64_t m = (cfg->strict || n <= size) ? n : size;
        if (cfg->strict && n != size) { o->status = OR_E_SIZE; o->reply_err = 1; }
        else if (ptr < region_base || m > region_bytes || ptr - region_base > region_bytes - m) {
          o->status = OR_E_PTR; o->reply_err = 1;
        } else {
          uint64_t b;
          for (b = 0; b < m; ++b) region[ptr - region_base + b] = L[c.off[1] + b];
          o->reply_err = 0;
        }
        {
          uint8_t tmp[32];
          uint64_t ln = or_rpc_put_reply_header(tmp, 0, c.xid), wl;
          ln = or_xdr_put_u32(tmp, ln, (uint32_t)o->reply_err);
          wl = or_frame_wire_size(ln, F);
          if (send_rings) {
            uint8_t* wire = (uint8_t*)malloc(wl);
            uint64_t b;
            or_frame_record(tmp, ln, F, wire);
            for (b = 0; b < wl; ++b) send_rings[r][(w + b) & (send_caps[r] - 1)] = wire[b];
            free(wire);
          }
          o->reply_off = w;
          o->reply_wire = wl;
          w += wl;
        }
      } else if (o->status == OR_OK && c.proc == cfg->proc_d2h) {
        uint64_t ptr = c.value[0], size = c.value[1], wl;
        const uint8_t* src = 0;
        if (size > 0xffffffffull || ptr < region_base || size > region_bytes || ptr - region_base > region_bytes - size) {
          o->status = OR_E_PTR; o->reply_err = 1; size = 0;
        } else {
          o->reply_err = 0;
          src = region + (ptr - region_base);
        }
        wl = or_encode_memcpy_d2h(c.xid, src, (uint32_t)size, o->reply_err, F, 0);
        if (send_rings) {
          uint8_t* wire = (uint8_t*)malloc(wl);
          uint64_t b;
          or_encode_memcpy_d2h(c.xid, src, (uint32_t)size, o->reply_err, F, wire);
          for (b = 0; b < wl; ++b) send_rings[r][(w + b) & (send_caps[r] - 1)] = wire[b];
          free(wire);
        }
        o->reply_off = w;
        o->reply_wire = wl;
        w += wl;
      }
      total++;
      free(L);
    }
    reply_bytes[r] = w - out_off[r];
  }
  }
  *n_out = total;
  free(schemas); free(frags); free(recs); free(seen_xid); free(xid_readable); free(parents);
  return OR_OK;
}
