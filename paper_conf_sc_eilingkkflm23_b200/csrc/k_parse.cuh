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

// The checks run on all 32 lanes in lockstep (every value they branch on is warp-uniform): lane k holds word k
// of the warp's head / tail buffer (hw), and a 4-byte-aligned read of either comes by shuffle from its lane,
// so the dependent chain per word is a shuffle instead of a generic shared-memory load.
struct Parser {
  LogicalRecord L;
  uint64_t o;           // always a multiple of 4 (every XDR item is)
  const uint8_t* head;  // first `nhead` logical bytes, already in shared memory
  uint32_t nhead;
  const uint8_t* tail;  // logical bytes [tail_lo, L.len), already in shared memory (tail_lo == L.len: none)
  uint64_t tail_lo;
  uint32_t hw;          // this lane's word of head (lanes 0-15) / tail (lanes 16-31), as stored
  __device__ __forceinline__ uint8_t byte(uint64_t at) {
    return at < nhead ? head[at] : (at >= tail_lo && at < L.len) ? tail[at - tail_lo] : L.byte(at);
  }
  __device__ int get_u32(uint32_t& v) {
    if (o + 4 > L.len) return CRK_E_TRUNCATED;
    int src = -1;
    if (o + 4 <= nhead) src = (int)(o >> 2);
    else if (o >= tail_lo && !((o - tail_lo) & 3)) src = (int)(kHead / 4 + ((o - tail_lo) >> 2));
    const uint32_t w = __shfl_sync(0xffffffffu, hw, src < 0 ? 0 : src);
    if (src >= 0) {
      v = __byte_perm(w, 0, 0x0123);  // big-endian
    } else if (o >= tail_lo) {
      const uint8_t* b = tail + (o - tail_lo);
      v = ((uint32_t)b[0] << 24) | ((uint32_t)b[1] << 16) | ((uint32_t)b[2] << 8) | b[3];
    } else {
      v = L.be32(o);
    }
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

// Parse of dense record d (ring `ring`, index slot `slot`) by one warp: the lanes run the checks in the
// oracle's order in lockstep (Parser), lane k keeps item k's fields, and the record's fields and the xid table
// entry are written at the end; head_buf is the warp's kHeadBuf-byte shared buffer for the record head.
// Used by K3 (one warp per record), the fused front end and the persistent server (warp-uniform calls).
// `sole`: d is the step's only record, so its xid goes into the (cleared) table with a plain store instead
// of a compare-and-swap whose result the warp would wait for.
__device__ void parse_record(const IndexDev& ix, const SchemaTable& sch, const ConfigDev& cfg, uint32_t d,
                             uint32_t ring, uint32_t slot, uint8_t* head_buf, uint32_t lane, bool sole = false,
                             uint64_t prefetch_max = 0) {
  STEP_MARK(lane == 0 && d == 0, 8, 0);
  Parser P;
  P.L.init(ix, ix.rings[ring], slot);
  P.o = 0;
  STEP_MARK(lane == 0 && d == 0, 9, P.L.len ^ P.L.nfrags ^ P.L.frag0 ^ P.L.R.mask);
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
  STEP_MARK(lane == 0 && d == 0, 10, ntail ^ ph_last ^ P.L.phys[0]);
  // prefetch_max (the persistent server, device-memory rings): a record of at most that many bytes has its first
  // fragment pulled into L2 now (a hint: no registers, nothing waits), so the move that follows the planning
  // reads the payload from L2 instead of HBM
  if (prefetch_max && lane == 0 && P.L.len <= prefetch_max) {
    uint64_t c = P.L.phys[0] & ~15ull;
    const uint64_t e = (P.L.phys[0] + n0 + 15) & ~15ull;
    while (c < e) {
      const uint64_t o = c & P.L.R.mask, room = P.L.R.mask + 1 - o, left = e - c;
      const uint32_t n = (uint32_t)(room < left ? room : left);
      asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(P.L.R.base + o), "r"(n) : "memory");
      c += n;
    }
  }
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
  P.hw = reinterpret_cast<const uint32_t*>(head_buf)[lane];
  STEP_MARK(lane == 0 && d == 0, 11, P.hw);
  const bool strict = cfg.strict != 0;
  uint32_t xid = 0, proc = 0, v, nitems = 0;
  int st = CRK_OK;
  uint32_t my_kind = 0;  // lane k: item k's fields
  uint64_t my_off = 0, my_cnt = 0, my_val = 0;
  // The fixed-layout head (RFC 5531 §9 call_body with zero-length cred and verf bodies, the AUTH_NONE case):
  // its ten words sit in lanes 0-9, so the four header checks run on four lanes at once.  When they all
  // pass and both auth lengths are 0 the sequential checks would reach offset 40 with these values; any
  // other head takes the sequential path from offset 0 (same checks, same first failure).
  const uint32_t wv = __byte_perm(P.hw, 0, 0x0123);
  const uint32_t expect = lane == 1 ? 0u : lane == 2 ? 2u : lane == 3 ? cfg.prog : cfg.vers;
  const bool fixed_ok = P.nhead >= 40 &&
                        !__ballot_sync(0xffffffffu, lane >= 1 && lane <= 4 && wv != expect) &&
                        __shfl_sync(0xffffffffu, wv, 7) == 0 && __shfl_sync(0xffffffffu, wv, 9) == 0;
  do {
    if (fixed_ok) {
      xid = __shfl_sync(0xffffffffu, wv, 0);
      proc = __shfl_sync(0xffffffffu, wv, 5);
      P.o = 40;
    } else {
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
    }
    // the first schema entry of the procedure (two entries per lane cover kMaxProcs <= 64)
    static_assert(kMaxProcs <= 64, "two schema entries per lane");
    const uint32_t hit_lo = __ballot_sync(0xffffffffu, lane < sch.n && sch.s[lane].proc == proc);
    const uint32_t hit_hi = __ballot_sync(0xffffffffu, lane + 32 < sch.n && sch.s[lane + 32].proc == proc);
    if (!hit_lo && !hit_hi) { st = CRK_E_PROC; break; }
    const Schema& sc = sch.s[hit_lo ? __ffs(hit_lo) - 1 : 32 + __ffs(hit_hi) - 1];
    if (!fixed_ok) {
      if ((st = P.get_auth(strict))) break;           // cred
      if ((st = P.get_auth(strict))) break;           // verf
    }
    nitems = sc.n_items;
    // Closed forms for the two memcpy schemas (built-in HtoD: u64, opaque<>, u64; DtoH: u64, u64) after the
    // fixed-layout head, taken only when every check of the item loop below would pass: the record ends exactly
    // after the last item, each word it reads sits in the warp's head / tail buffer, and (strict) the opaque's
    // pad bytes are zero.  The offsets, counts and values are then the loop's (RFC 4506 §4.5 hyper, §4.10
    // opaque<>); any other record takes the loop, which finds the first failing check in the oracle's order.
    bool closed = false;
    if (fixed_ok) {
      const bool h2d = nitems == 3 && sc.items[0] == CRK_K_U64 && sc.items[1] == CRK_K_OPAQUE_VAR &&
                       sc.items[2] == CRK_K_U64;
      const bool d2h = nitems == 2 && sc.items[0] == CRK_K_U64 && sc.items[1] == CRK_K_U64;
      const uint64_t len = P.L.len;
      // the buffer lane holding the aligned word at logical offset at (get_u32's mapping), -1: not buffered
      auto word_src = [&](uint64_t at) -> int {
        if (at + 4 <= P.nhead) return (int)(at >> 2);
        if (at >= P.tail_lo && at + 4 <= len && !((at - P.tail_lo) & 3)) return (int)(kHead / 4 + ((at - P.tail_lo) >> 2));
        return -1;
      };
      auto buffered_byte = [&](uint64_t at, bool& ok) -> uint8_t {
        if (at < P.nhead) return P.head[at];
        if (at >= P.tail_lo && at < len) return P.tail[at - P.tail_lo];
        ok = false;
        return 0;
      };
      const uint32_t w10 = __shfl_sync(0xffffffffu, wv, 10), w11 = __shfl_sync(0xffffffffu, wv, 11);
      const uint32_t w12 = __shfl_sync(0xffffffffu, wv, 12), w13 = __shfl_sync(0xffffffffu, wv, 13);
      if (h2d && P.nhead >= 52) {
        const uint64_t c = w12, pn = pad4(c), o2 = 52 + c + pn;
        const int s0 = word_src(o2), s1 = word_src(o2 + 4);
        bool ok = o2 + 8 == len && s0 >= 0 && s1 >= 0;
        if (ok && strict)
          for (uint64_t i = 0; i < pn; ++i) {
            bool av = true;
            const uint8_t b = buffered_byte(52 + c + i, av);
            ok = ok && av && b == 0;
          }
        const uint32_t z0 = __byte_perm(__shfl_sync(0xffffffffu, P.hw, s0 < 0 ? 0 : s0), 0, 0x0123);
        const uint32_t z1 = __byte_perm(__shfl_sync(0xffffffffu, P.hw, s1 < 0 ? 0 : s1), 0, 0x0123);
        if (ok) {
          closed = true;
          my_kind = lane == 1 ? (uint32_t)CRK_K_OPAQUE_VAR : (uint32_t)CRK_K_U64;
          my_off = lane == 0 ? 40 : lane == 1 ? 52 : o2;
          my_cnt = lane == 1 ? c : 0;
          my_val = lane == 0 ? ((uint64_t)w10 << 32 | w11) : lane == 2 ? ((uint64_t)z0 << 32 | z1) : 0;
        }
      } else if (d2h && P.nhead >= 56 && len == 56) {
        closed = true;
        my_kind = CRK_K_U64;
        my_off = lane == 0 ? 40 : 48;
        my_cnt = 0;
        my_val = lane == 0 ? ((uint64_t)w10 << 32 | w11) : ((uint64_t)w12 << 32 | w13);
      }
    }
    if (closed) break;
    const uint32_t my_item = lane < nitems ? sc.items[lane] : 0;
    for (uint32_t it = 0; it < nitems && st == CRK_OK; ++it) {
      const uint32_t code = __shfl_sync(0xffffffffu, my_item, it);
      const uint32_t kind = code & 0xff, fixed = code >> 8, es = elem_size(kind);
      uint64_t o_it = 0, c_it = 0, v_it = 0;
      if (kind == CRK_K_U32) {
        st = P.get_u32(v);
        o_it = P.o - 4;
        v_it = v;
      } else if (kind == CRK_K_U64) {
        uint32_t hi32 = 0, lo32 = 0;                  // RFC 4506 §4.5: most significant word first
        if (!(st = P.get_u32(hi32))) st = P.get_u32(lo32);
        o_it = P.o - 8;
        v_it = ((uint64_t)hi32 << 32) | lo32;
      } else {
        uint64_t c = fixed;
        if (kind_is_var(kind)) {
          st = P.get_u32(v);
          c = v;
        }
        if (st == CRK_OK) {
          const uint64_t bytes = c * es, pn = pad4(bytes);
          if (P.o + bytes + pn > P.L.len) st = CRK_E_TRUNCATED;
          else if (strict && !P.pad_is_zero(P.o + bytes, pn)) st = CRK_E_PAD;
          else {
            o_it = P.o;
            c_it = c;
            P.o += bytes + pn;
          }
        }
      }
      if (lane == it) {
        my_kind = kind;
        my_off = o_it;
        my_cnt = c_it;
        my_val = v_it;
      }
    }
    if (st != CRK_OK) break;
    if (strict && P.o != P.L.len) st = CRK_E_TRAILING;
  } while (0);
  STEP_MARK(lane == 0 && d == 0, 12, st ^ nitems);
  if (lane < nitems) {  // the items parsed before any failure; the tables are read only for OK / E_TRAILING
    const uint64_t k = (uint64_t)d * kMaxItems + lane;
    ix.p_kind[k] = my_kind;
    ix.p_off[k] = my_off;
    ix.p_count[k] = my_cnt;
    ix.p_value[k] = my_val;
  }
  if (lane != 0) return;
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
