// K3: CALL parse (RFC 5531 §9, opaque_auth §8.2) and arguments by schema (RFC 4506), one warp per
// record, plus the xid -> record lookup table (reading R11: the earliest record owns an xid).
// The check order is the oracle's (oracle/oracle.c or_parse_call), so the first failure in logical
// order is the record's wire status.
#pragma once
#include "crk_device.cuh"
#include "crk_logical.cuh"

namespace crk {

namespace {

constexpr uint32_t kAuthMax = 400;  // RFC 5531 §8.2 opaque body<400>

__device__ __forceinline__ uint32_t elem_size(uint32_t kind) {
  switch (kind) {
    case CRK_K_OPAQUE_VAR: case CRK_K_OPAQUE_FIX: return 1;
    case CRK_K_I32_VAR: case CRK_K_U32_VAR: case CRK_K_F32_VAR:
    case CRK_K_I32_FIX: case CRK_K_U32_FIX: case CRK_K_F32_FIX: return 4;
    case CRK_K_I64_VAR: case CRK_K_U64_VAR: case CRK_K_F64_VAR:
    case CRK_K_I64_FIX: case CRK_K_U64_FIX: case CRK_K_F64_FIX: return 8;
    default: return 0;
  }
}
__device__ __forceinline__ bool kind_is_var(uint32_t k) {
  return k == CRK_K_OPAQUE_VAR || (k >= CRK_K_I32_VAR && k <= CRK_K_F64_VAR);
}

constexpr uint32_t kHead = 64;  // record head prefetched by the warp (CALL header + memcpy args)
constexpr uint32_t kTail = 64;  // record tail prefetched with it (the arguments after a bulk opaque<>)
constexpr uint32_t kHeadBuf = kHead + kTail;  // per-warp shared buffer

struct Parser {
  LogicalRecord L;
  uint64_t o;
  const uint8_t* head;  // first `nhead` logical bytes, already in shared memory
  uint32_t nhead;
  const uint8_t* tail;  // logical bytes [tail_lo, L.len), already in shared memory (tail_lo == L.len: none)
  uint64_t tail_lo;
  __device__ __forceinline__ uint8_t byte(uint64_t at) {
    return at < nhead ? head[at] : (at >= tail_lo && at < L.len) ? tail[at - tail_lo] : L.byte(at);
  }
  __device__ int get_u32(uint32_t& v) {
    if (o + 4 > L.len) return CRK_E_TRUNCATED;
    const uint8_t* b = o + 4 <= nhead ? head + o : o >= tail_lo ? tail + (o - tail_lo) : nullptr;
    if (b && !(reinterpret_cast<uintptr_t>(b) & 3))  // one shared-memory word, byte-swapped (big-endian)
      v = __byte_perm(*reinterpret_cast<const uint32_t*>(b), 0, 0x0123);
    else if (b)
      v = ((uint32_t)b[0] << 24) | ((uint32_t)b[1] << 16) | ((uint32_t)b[2] << 8) | b[3];
    else
      v = L.be32(o);
    o += 4;
    return CRK_OK;
  }
  // RFC 4506 §3: the pad bytes after an item must be zero (checked in strict mode)
  __device__ bool pad_is_zero(uint64_t at, uint64_t n) {
    for (uint64_t i = 0; i < n; ++i)
      if (byte(at + i) != 0) return false;
    return true;
  }
  __device__ int get_auth(bool strict) {
    uint32_t flavor, len;
    int st;
    if ((st = get_u32(flavor))) return st;
    if ((st = get_u32(len))) return st;
    if (len > kAuthMax) return CRK_E_AUTH;
    if (o + len + pad4(len) > L.len) return CRK_E_TRUNCATED;
    if (strict && !pad_is_zero(o + len, pad4(len))) return CRK_E_PAD;
    o += len + pad4(len);
    return CRK_OK;
  }
};

// Parse of dense record d (ring `ring`, index slot `slot`) by one warp: lane 0 runs the checks in the
// oracle's order and writes the parsed-call tables and the xid table; head_buf is the warp's kHeadBuf-byte
// shared buffer for the record head.  Used by K3 (one warp per record) and by the persistent server.
// `sole`: d is the step's only record, so its xid goes into the (cleared) table with a plain store instead
// of a compare-and-swap whose result the warp would wait for.
__device__ void parse_record(const IndexDev& ix, const SchemaTable& sch, const ConfigDev& cfg, uint32_t d,
                             uint32_t ring, uint32_t slot, uint8_t* head_buf, uint32_t lane, bool sole = false) {
  Parser P;
  P.L.init(ix, ix.rings[ring], slot);
  P.o = 0;
  // the warp prefetches, in one round trip, the record head from its first fragment and the record tail
  // from its last fragment (when the tail lies inside it): a memcpy CALL's header, pointer, opaque length
  // and, after the bulk data, its pad and size argument
  const uint64_t n0 = P.L.flen(0);
  const uint64_t nh = n0 < P.L.len ? n0 : P.L.len;
  P.nhead = nh < kHead ? (uint32_t)nh : kHead;
  const uint32_t kl = P.L.nfrags - 1;
  const uint64_t ls_last = P.L.lstart[kl], ph_last = P.L.phys[kl];
  // the tail window starts at most kTail bytes before the end, inside the last fragment and past the head
  const uint64_t want = P.L.len > kTail ? P.L.len - kTail : 0;
  const uint64_t tlo = max(max(want, (uint64_t)P.nhead), ls_last);
  P.tail_lo = P.L.len > tlo ? tlo : P.L.len;
  const uint32_t ntail = (uint32_t)(P.L.len - P.tail_lo);
  P.head = head_buf;
  P.tail = head_buf + kHead;
  uint8_t b[4];
  b[0] = lane < P.nhead ? ring_byte(P.L.R, P.L.phys[0] + lane) : 0;
  b[1] = lane + 32 < P.nhead ? ring_byte(P.L.R, P.L.phys[0] + lane + 32) : 0;
  b[2] = lane < ntail ? ring_byte(P.L.R, ph_last + (P.tail_lo - ls_last) + lane) : 0;
  b[3] = lane + 32 < ntail ? ring_byte(P.L.R, ph_last + (P.tail_lo - ls_last) + lane + 32) : 0;
  head_buf[lane] = b[0];
  head_buf[lane + 32] = b[1];
  head_buf[kHead + lane] = b[2];
  head_buf[kHead + lane + 32] = b[3];
  __syncwarp();
  if (lane != 0) return;
  const bool strict = cfg.strict != 0;
  uint32_t xid = 0, proc = 0, v, nitems = 0;
  int st = CRK_OK;
  const Schema* sc = nullptr;
  uint64_t* off = ix.p_off + (uint64_t)d * kMaxItems;
  uint64_t* cnt = ix.p_count + (uint64_t)d * kMaxItems;
  uint64_t* val = ix.p_value + (uint64_t)d * kMaxItems;
  uint32_t* kinds = ix.p_kind + (uint64_t)d * kMaxItems;
  do {
    if ((st = P.get_u32(xid))) break;
    if ((st = P.get_u32(v))) break;
    if (v != 0) { st = CRK_E_RPC; break; }          // msg_type CALL
    if ((st = P.get_u32(v))) break;
    if (v != 2) { st = CRK_E_RPC; break; }          // rpcvers 2
    if ((st = P.get_u32(v))) break;
    if (v != cfg.prog) { st = CRK_E_RPC; break; }
    if ((st = P.get_u32(v))) break;
    if (v != cfg.vers) { st = CRK_E_RPC; break; }
    if ((st = P.get_u32(proc))) break;
    for (uint32_t i = 0; i < sch.n; ++i)
      if (sch.s[i].proc == proc) { sc = &sch.s[i]; break; }
    if (!sc) { st = CRK_E_PROC; break; }
    if ((st = P.get_auth(strict))) break;           // cred
    if ((st = P.get_auth(strict))) break;           // verf
    nitems = sc->n_items;
    for (uint32_t it = 0; it < sc->n_items && st == CRK_OK; ++it) {
      const uint32_t kind = sc->items[it] & 0xff, fixed = sc->items[it] >> 8, es = elem_size(kind);
      kinds[it] = kind;
      cnt[it] = 0;
      val[it] = 0;
      if (kind == CRK_K_U32) {
        if ((st = P.get_u32(v))) break;
        off[it] = P.o - 4;
        val[it] = v;
      } else if (kind == CRK_K_U64) {
        uint32_t hi32, lo32;                          // RFC 4506 §4.5: most significant word first
        if ((st = P.get_u32(hi32))) break;
        if ((st = P.get_u32(lo32))) break;
        off[it] = P.o - 8;
        val[it] = ((uint64_t)hi32 << 32) | lo32;
      } else {
        uint64_t c;
        if (kind_is_var(kind)) {
          if ((st = P.get_u32(v))) break;
          c = v;
        } else {
          c = fixed;
        }
        const uint64_t bytes = c * es, pn = pad4(bytes);
        if (P.o + bytes + pn > P.L.len) { st = CRK_E_TRUNCATED; break; }
        if (strict && !P.pad_is_zero(P.o + bytes, pn)) { st = CRK_E_PAD; break; }
        off[it] = P.o;
        cnt[it] = c;
        P.o += bytes + pn;
      }
    }
    if (st != CRK_OK) break;
    if (strict && P.o != P.L.len) st = CRK_E_TRAILING;
  } while (0);
  ix.p_slot[d] = slot;
  ix.p_frag0[d] = P.L.frag0;
  ix.p_nfrags[d] = P.L.nfrags;
  ix.p_flen0[d] = (uint32_t)P.L.F0;
  ix.p_ring[d] = ring;
  ix.p_xid[d] = xid;
  ix.p_proc[d] = proc;
  ix.p_status[d] = st;
  ix.p_nitems[d] = nitems;
  if (P.L.len >= 4) {  // xid readable: insert, the smallest dense id wins (reading R11)
    const unsigned long long key = ((unsigned long long)xid << 32) | d;
    uint32_t h = (xid * 0x9E3779B1u) & ix.hash_mask;
    if (sole) {
      ix.xid_hash[h] = key;
      return;
    }
    for (;;) {
      unsigned long long old = atomicCAS(ix.xid_hash + h, ~0ull, key);
      if (old == ~0ull) break;
      if ((uint32_t)(old >> 32) == xid) { atomicMin(ix.xid_hash + h, key); break; }
      h = (h + 1) & ix.hash_mask;
    }
  }
}

}  // namespace
}  // namespace crk
