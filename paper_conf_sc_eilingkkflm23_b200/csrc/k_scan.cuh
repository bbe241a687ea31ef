// K1 + K2 (fragment part): speculative record-marking scan (RFC 5531 §11) with the segmented prefix
// sum of fragment lengths that gives every fragment its logical start.
//
// The header chain is sequential (p[k+1] = p[k] + 4 + len[k]).  One CTA per ring walks it in rounds.
// From a known true header at p, the CTA splits into two groups, one per predicted header value h_g:
// thread u of group g reads the candidate header at p + u * (4 + len(h_g)).  If headers 0..u-1 all equal
// h_g their positions are exact, so candidate u is a true header (induction); the first u* whose value
// differs is still a true header.  The group with the longer run wins: a round accepts u* + 1 headers
// with one memory latency.  Predictor 0 follows the stride of multi-fragment records (greedy F-byte
// fragments); predictor 1 remembers the shape of the last single-fragment record, so streams that mix
// large HtoD calls with small DtoH calls advance about one record per round, and
// back-to-back identical records (C1) a whole group per round.  Because headers 0..u*-1 are identical,
// the fragment lengths' segmented prefix sums (logical starts) and the record boundaries have closed
// forms in u; the checks are then the oracle's, in its order (oracle/oracle.c or_frame_scan;
// DESIGN.md §3 readings R1, R2, R8): E_FRAG -> INCOMPLETE (data past tail) -> index capacity.
#pragma once
#include "crk_device.cuh"

namespace crk {

namespace {

enum : uint32_t { STOP_NONE = 0, STOP_FRAG = 1, STOP_INCOMPLETE = 2, STOP_CAP = 3 };
constexpr uint32_t kNoPred = 0xffffffffu;  // a predictor value no header is expected to match
constexpr uint32_t kJ = 4;                 // candidate headers per thread and CTA round (independent loads)
constexpr uint32_t kWJ = 2;                // candidate headers per lane and warp round
constexpr uint32_t kWTT = 16 * kWJ;        // candidates per group and warp round (16 lanes per group)
constexpr uint32_t kChase = 4096;          // max headers per chase pass (irregular framing)
constexpr uint32_t kFull = 0xffffffffu;
constexpr uint64_t kChaseFirst = 16384;     // windows up to this many bytes start with a chase pass

#ifdef CRK_SCAN_TRACE
// Diagnostic build only (build.py build_trace -> lib/libcrk_trace.so): per ring, one entry per round /
// chase hop = clock64 at its end (low 40 bits) | mode (3 bits) << 40 | headers accepted << 43.
constexpr uint32_t kTraceRings = 64, kTraceLen = 4096;
__device__ unsigned long long g_scan_trace[kTraceRings][kTraceLen];
__device__ uint32_t g_scan_trace_n[kTraceRings];
__device__ __forceinline__ void trace(uint32_t mode, uint32_t n) {
  const uint32_t r = blockIdx.x;
  if (r >= kTraceRings) return;
  const uint32_t i = g_scan_trace_n[r];
  if (i < kTraceLen) {
    g_scan_trace[r][i] = (clock64() & ((1ull << 40) - 1)) | ((unsigned long long)mode << 40) |
                         ((unsigned long long)n << 43);
    g_scan_trace_n[r] = i + 1;
  }
}
#define SCAN_TRACE(writer, mode, n) \
  do {                              \
    if (writer) trace(mode, n);     \
  } while (0)
#else
#define SCAN_TRACE(writer, mode, n) \
  do {                              \
  } while (0)
#endif

struct ScanState {
  uint64_t p, r0, sum;
  uint32_t f0, nf, nr;
  uint32_t hp[2];
  uint32_t done;
  int32_t status;
  uint64_t consumed;
  uint32_t kept_frags;
  uint32_t wide;                      // CTA rounds (a long regular run) instead of warp rounds
  uint32_t gmin[32], gh[32], gv[32];  // per warp: first mismatch, its header, its validity
  uint32_t fmin[32], fcode[32];       // per warp: first failing check and its code
};

// The walk state between rounds (uniform across the lanes of warp 0 in the warp modes).
struct Walk {
  uint64_t p, r0, sum;
  uint32_t nf, nr, f0, hp0, hp1;
  bool stop;
  int32_t status;
  uint64_t consumed;
  uint32_t kept;
};

struct Env {
  IndexDev ix;
  RingDesc R;
  uint64_t max_record_bytes, fbase, rbase;
  uint32_t FC, RC;
};

// Header at cursor q, read as the aligned word(s) that contain it (any alignment, across the wrap); the
// second word only when q is not 4-aligned (framing with lengths that are multiples of 4 never needs it).
__device__ __forceinline__ void load_hdr(const RingDesc& R, uint64_t q, bool ok, uint32_t& w0, uint32_t& w1) {
  const uint64_t a = q & ~3ull;
  w0 = ok ? CRK_RO_LD(reinterpret_cast<const uint32_t*>(R.base + (a & R.mask))) : 0u;
  w1 = (ok && (q & 3)) ? CRK_RO_LD(reinterpret_cast<const uint32_t*>(R.base + ((a + 4) & R.mask))) : 0u;
}
__device__ __forceinline__ uint32_t join_hdr(uint64_t q, uint32_t w0, uint32_t w1) {
  return bswap32(__funnelshift_r(w0, w1, 8 * (uint32_t)(q & 3)));
}

// Index entries of fragment number nf (and of the record it completes).
__device__ __forceinline__ void emit_frag(const Env& E, uint32_t nf, uint64_t q, uint64_t len, uint32_t last,
                                          uint64_t send, bool start, uint64_t r0, uint32_t f0, uint32_t nrec) {
  const uint64_t fs = E.fbase + nf;
  E.ix.frag_phys[fs] = q + 4;
  E.ix.frag_lstart[fs] = send - len;
  E.ix.frag_hdr[fs] = (uint32_t)len | (last << 31);
  if (last) {
    const uint64_t rs = E.rbase + nrec;
    E.ix.rec_begin[rs] = start ? q : r0;
    E.ix.rec_len[rs] = send;
    E.ix.rec_frag0[rs] = (uint32_t)(E.fbase + (start ? nf : f0));
    E.ix.rec_nfrags[rs] = start ? 1u : nf - f0 + 1;
  }
}

// L2 prefetch of a ring span through the TMA unit (no registers, no completion to wait for).
__device__ __forceinline__ void prefetch_l2(const RingDesc& R, uint64_t c, uint32_t bytes) {
  const uint64_t o = c & R.mask, room = R.mask + 1 - o;
  const uint32_t n = room < bytes ? (uint32_t)room : bytes;
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(R.base + o), "r"(n) : "memory");
}

// The index work for a batch of consecutive chain hops, one per lane (lane k = hop k at cursor myq with
// header myh; hop 0 is at W.p, each next hop at the previous one's cursor + 4 + length): for the first
// n_take hops, the closed forms of or_frame_scan's loop -- segmented prefix sums of the lengths (logical
// starts), record boundaries -- and its checks in its order (E_FRAG -> INCOMPLETE -> index capacity),
// all with warp scans, then the fragment / record index entries of the hops before the first failing
// one.  On a failure the outcome is recorded in W (stop) and its hop number returned; otherwise W
// advances past hop n_take - 1 (and the predictors follow its headers) and -1 is returned.  Used by the
// chase pass below and by the chunked scan's emission (k_mscan.cu), whose hops come from a log.
__device__ int take_hops(const Env& E, Walk& W, uint32_t lane, uint32_t n_take, uint64_t myq, uint32_t myh) {
  const uint64_t tail = E.R.tail;
  const uint32_t vmask = n_take >= 32 ? kFull : (1u << n_take) - 1;
  const bool v = lane < n_take;
  const uint64_t len = v ? (uint64_t)(myh & 0x7fffffffu) : 0ull;
  const uint32_t last = v ? myh >> 31 : 0u;
  const uint32_t lastm = __ballot_sync(kFull, last);
  const uint32_t startm = ((lastm << 1) | (W.p == W.r0 ? 1u : 0u)) & vmask;
  const bool start = (startm >> lane) & 1;
  uint64_t P = len;  // inclusive prefix of lengths over the batch
#pragma unroll
  for (uint32_t o = 1; o < 32; o <<= 1) {
    const uint64_t y = __shfl_up_sync(kFull, P, o);
    if (lane >= o) P += y;
  }
  const uint64_t Ex = P - len;
  const uint32_t below = startm & (lane == 31 ? kFull : (2u << lane) - 1);
  const int j = below ? 31 - __clz(below) : -1;  // this hop's record began at hop j of the batch
  const uint64_t Ej = __shfl_sync(kFull, Ex, j < 0 ? 0 : j);
  const uint64_t qj = __shfl_sync(kFull, myq, j < 0 ? 0 : j);
  const uint64_t send = j >= 0 ? P - Ej : W.sum + P;  // logical end of this fragment in its record
  const uint64_t rbeg = j >= 0 ? qj : W.r0;
  const uint32_t f0 = j >= 0 ? W.nf + (uint32_t)j : W.f0;
  const uint32_t nrec = W.nr + __popc(lastm & ((1u << lane) - 1));
  uint32_t code = STOP_NONE;
  if (v) {
    if (send > E.max_record_bytes) code = STOP_FRAG;
    else if (myq + 4 + len > tail) code = STOP_INCOMPLETE;
    else if (W.nf + lane >= E.FC || (start && nrec >= E.RC)) code = STOP_CAP;
  }
  const uint32_t failm = __ballot_sync(kFull, code != STOP_NONE);
  const uint32_t tf = failm ? __ffs(failm) - 1 : 32u;
  const uint32_t n_acc = tf < n_take ? tf : n_take;
  if (lane < n_acc) {
    const uint64_t fs = E.fbase + W.nf + lane;
    E.ix.frag_phys[fs] = myq + 4;
    E.ix.frag_lstart[fs] = send - len;
    E.ix.frag_hdr[fs] = myh;
    // (nrec < RC always holds for a walk that checks every record start; a chunk of the chunked scan that
    // starts inside a record after an earlier chunk's capacity stop must still stay inside the slice)
    if (last && nrec < E.RC) {
      const uint64_t rs = E.rbase + nrec;
      E.ix.rec_begin[rs] = start ? myq : rbeg;
      E.ix.rec_len[rs] = send;
      E.ix.rec_frag0[rs] = (uint32_t)(E.fbase + f0);
      E.ix.rec_nfrags[rs] = W.nf + lane - f0 + 1;
    }
  }
  if (tf < n_take) {  // hop tf's check failed: the outcome is recorded there
    const uint32_t c = __shfl_sync(kFull, code, tf);
    const uint32_t nr_t = __shfl_sync(kFull, nrec, tf);
    const bool st_t = (startm >> tf) & 1;
    W.consumed = st_t ? __shfl_sync(kFull, myq, tf) : __shfl_sync(kFull, rbeg, tf);
    W.kept = st_t ? W.nf + tf : __shfl_sync(kFull, f0, tf);
    W.nr = nr_t;
    W.status = c == STOP_FRAG ? CRK_E_FRAG : c == STOP_INCOMPLETE ? CRK_INCOMPLETE
             : (nr_t > 0 ? CRK_INCOMPLETE : CRK_E_CAPACITY);
    W.stop = true;
    return (int)tf;
  }
  if (n_acc) {  // advance the state to after hop n_acc - 1 and update the predictors
    const uint32_t L = n_acc - 1, am = n_acc >= 32 ? kFull : (1u << n_acc) - 1;
    const uint64_t qL = __shfl_sync(kFull, myq, L), lenL = __shfl_sync(kFull, len, L);
    const uint64_t sendL = __shfl_sync(kFull, send, L), rbegL = __shfl_sync(kFull, rbeg, L);
    const uint32_t f0L = __shfl_sync(kFull, f0, L), nrecL = __shfl_sync(kFull, nrec, L);
    const uint32_t hL = __shfl_sync(kFull, myh, L);
    const uint32_t singlem = __ballot_sync(kFull, start && last) & am, nonlastm = ~lastm & am;
    if (singlem) W.hp1 = __shfl_sync(kFull, myh, 31 - __clz(singlem));
    if (nonlastm) W.hp0 = __shfl_sync(kFull, myh, 31 - __clz(nonlastm));
    W.p = qL + 4 + lenL;
    W.nf += n_acc;
    if (hL >> 31) {
      W.nr = nrecL + 1;
      W.r0 = W.p;
      W.sum = 0;
      W.f0 = W.nf;
    } else {
      W.nr = nrecL;
      W.sum = sendL;
      W.r0 = rbegL;
      W.f0 = f0L;
    }
  }
  return -1;
}

// Chase pass: the serial walk of the chain, for framing no predictor follows.  It runs in batches of 32
// hops.  The walk itself carries only the chain (p -> p + 4 + len(be32(p))): every lane follows it
// (broadcast loads) and lane k keeps hop k's cursor and header.  All per-header work is then take_hops
// for the 32 hops at once, so a hop costs one load latency.  Hops past a failing header are walked but
// discarded (reads stay inside the ring).  Once a pass is long (an irregular stream), the TMA prefetches
// the ring ahead of the walk into L2 (kPfLead bytes ahead), so header reads hit L2 instead of HBM / the
// host link.  Stops after kChase headers, at a stop, or at two equal consecutive headers (a regular run
// the predictors can take over again).
#ifndef CRK_PF_LEAD
#define CRK_PF_LEAD (1ull << 20)  // prefetch frontier lead over the walk (bytes; 0 = no prefetch)
#endif
#ifndef CRK_PF_CHUNK
#define CRK_PF_CHUNK 65536u       // bytes per prefetch instruction (power of 2)
#endif
constexpr uint64_t kPfLead = CRK_PF_LEAD;
constexpr uint32_t kPfChunk = CRK_PF_CHUNK;
__device__ void chase(const Env& E, Walk& W, uint32_t lane) {
  const uint64_t tail = E.R.tail;
  uint32_t prev = kNoPred;
  uint64_t pf = 0;  // prefetch frontier (cursor), from the second batch of a pass on
  for (uint32_t b = 0; b < kChase / 32; ++b) {
    if (b == 1) pf = W.p & ~15ull;  // a long pass: start prefetching
    // ---- walk up to 32 hops
    uint64_t q = W.p, myq = 0;
    uint32_t myh = 0, n = 0, hw = prev;
#pragma unroll 1
    for (; n < 32; ++n) {
      if (q + 4 > tail) break;
      if (CRK_PF_LEAD && b && lane == 0) {
        const uint64_t want = min(q + kPfLead, tail);
        for (uint32_t i = 0; i < 4 && pf < want; ++i) {
          prefetch_l2(E.R, pf, kPfChunk);
          pf += kPfChunk - (pf & (kPfChunk - 1));  // chunks aligned to kPfChunk (never cross the wrap)
        }
      }
      const uint64_t a = q & ~3ull;
      const uint32_t w0 = CRK_RO_LD(reinterpret_cast<const uint32_t*>(E.R.base + (a & E.R.mask)));
      const uint32_t w1 = CRK_RO_LD(reinterpret_cast<const uint32_t*>(E.R.base + ((a + 4) & E.R.mask)));
      const uint32_t h = join_hdr(q, w0, w1);
      if (lane == n) { myq = q; myh = h; }
      q += 4 + (uint64_t)(h & 0x7fffffffu);
      if (h == hw) { ++n; break; }  // two equal headers: the batch ends here (the rounds take over)
      hw = h;
    }
    SCAN_TRACE(lane == 0, 2, n);
    const uint32_t hprev = __shfl_up_sync(kFull, myh, 1);
    const uint32_t eqm = __ballot_sync(kFull, lane < n && myh == (lane ? hprev : prev));
    const uint32_t te = eqm ? __ffs(eqm) - 1 : 32u;
    const uint32_t n_take = te < n ? te + 1 : n;
    if (take_hops(E, W, lane, n_take, myq, myh) >= 0) return;
    if (n_take) prev = __shfl_sync(kFull, myh, n_take - 1);
    if (te < n) return;  // two equal headers: back to the speculative rounds
    if (n < 32) {        // no readable header at W.p: the window ends here
      const bool st = W.p == W.r0;
      W.status = (st && W.p == tail) ? CRK_OK : CRK_INCOMPLETE;
      W.consumed = W.r0;
      W.kept = st ? W.nf : W.f0;
      W.stop = true;
      return;
    }
  }
}

// Warp rounds: the CTA round's speculation (two predictor groups, first mismatch still a true header,
// closed forms in u) on the 32 lanes of one warp -- 16 lanes x kWJ candidates per group -- with warp
// reductions instead of block barriers, so a round costs one memory latency.  Records that are not
// long regular runs (mixed HtoD / DtoH calls, small calls) are scanned here.  Returns true when a round
// matched every candidate (a long regular run: hand over to the CTA rounds); false on a stop.  After
// two rounds that accepted at most 2 headers each, a chase pass takes over.
__device__ bool warp_rounds(const Env& E, Walk& W, uint32_t lane) {
  const uint32_t grp = lane >> 4, u = lane & 15;
  // a short window (a few small calls) starts with a chase pass: one load per header and no speculation round
  // (whose candidates past a one-record window are all misses); the rounds take over at a regular run
  uint32_t miss = E.R.tail - W.p <= kChaseFirst ? 2u : 0u;
  for (;;) {
    if (miss >= 2) {
      chase(E, W, lane);
      if (W.stop) return false;
      miss = 0;
      continue;
    }
    const uint64_t p = W.p, r0 = W.r0, sum = W.sum;
    const uint32_t nf = W.nf, nr = W.nr, f0 = W.f0;
    const uint32_t hmine = grp ? W.hp1 : W.hp0;
    const uint64_t smine = 4 + (uint64_t)(hmine & 0x7fffffffu);
    uint32_t w0[kWJ], w1[kWJ];
    bool vv[kWJ];
#pragma unroll
    for (uint32_t j = 0; j < kWJ; ++j) {
      const uint64_t q = p + (uint64_t)(u + 16 * j) * smine;
      vv[j] = q + 4 <= E.R.tail;
      load_hdr(E.R, q, vv[j], w0[j], w1[j]);
    }
    uint32_t first_bad = kWTT, bh = 0, bv = 0;
#pragma unroll
    for (uint32_t j = 0; j < kWJ; ++j) {
      const uint32_t t = u + 16 * j;
      const uint32_t h = join_hdr(p + (uint64_t)t * smine, w0[j], w1[j]);
      if (first_bad == kWTT && !(vv[j] && h == hmine)) { first_bad = t; bh = h; bv = vv[j]; }
    }
    const uint32_t ts0 = __reduce_min_sync(kFull, grp == 0 ? first_bad : kWTT);
    const uint32_t ts1 = __reduce_min_sync(kFull, grp == 1 ? first_bad : kWTT);
    const uint32_t win = ts1 > ts0, tstar = win ? ts1 : ts0;
    SCAN_TRACE(lane == 0, 4, 0);  // candidate loads consumed
    uint32_t hstar = 0, vstar = 1;
    if (tstar < kWTT) {
      const uint32_t own = __ffs(__ballot_sync(kFull, grp == win && first_bad == tstar)) - 1;
      hstar = __shfl_sync(kFull, bh, own);
      vstar = __shfl_sync(kFull, bv, own);
    }
    const uint32_t hp = win ? W.hp1 : W.hp0;
    const uint64_t Lp = hp & 0x7fffffffu, stride = 4 + Lp;
    const uint32_t lastp = hp >> 31;
    const bool end_at_star = tstar < kWTT && !vstar;
    const uint32_t n_hdr = tstar == kWTT ? kWTT : (end_at_star ? tstar : tstar + 1);
    // closed forms of header t (headers 0..tstar-1 equal hp)
    auto at = [&](uint32_t t, uint64_t& q, uint64_t& len, uint32_t& last, bool& start, uint64_t& send,
                  uint32_t& nrec) {
      q = p + (uint64_t)t * stride;
      len = t < tstar ? Lp : (uint64_t)(hstar & 0x7fffffffu);
      last = t < tstar ? lastp : (hstar >> 31);
      start = t == 0 ? (p == r0) : (lastp != 0);
      if (!lastp) send = sum + (uint64_t)t * Lp + len;
      else send = t == 0 ? (start ? len : sum + len) : len;
      nrec = lastp ? nr + t : nr;
    };
    uint32_t first_fail = kFull, my_code = STOP_NONE;
#pragma unroll
    for (uint32_t j = 0; j < kWJ; ++j) {
      const uint32_t t = u + 16 * j;
      if (grp != win || t >= n_hdr || first_fail != kFull) continue;
      uint64_t q, len, send;
      uint32_t last, nrec;
      bool start;
      at(t, q, len, last, start, send, nrec);
      uint32_t code = STOP_NONE;
      if (send > E.max_record_bytes) code = STOP_FRAG;
      else if (q + 4 + len > E.R.tail) code = STOP_INCOMPLETE;
      else if (nf + t >= E.FC || (start && nrec >= E.RC)) code = STOP_CAP;
      if (code != STOP_NONE) { first_fail = t; my_code = code; }
    }
    const uint32_t tf = __reduce_min_sync(kFull, first_fail);
    uint32_t code_f = STOP_NONE;
    if (tf != kFull) code_f = __shfl_sync(kFull, my_code, __ffs(__ballot_sync(kFull, first_fail == tf)) - 1);
    const uint32_t n_emit = tf < n_hdr ? tf : n_hdr;
#pragma unroll
    for (uint32_t j = 0; j < kWJ; ++j) {
      const uint32_t t = u + 16 * j;
      if (grp != win || t >= n_emit) continue;
      uint64_t q, len, send;
      uint32_t last, nrec;
      bool start;
      at(t, q, len, last, start, send, nrec);
      emit_frag(E, nf + t, q, len, last, send, start, r0, f0, nrec);
    }
    uint64_t q, len, send;
    uint32_t last, nrec;
    bool start;
    if (tf < n_hdr || end_at_star) {  // the stopping header records the outcome
      const uint32_t t = tf < n_hdr ? tf : tstar;
      at(t, q, len, last, start, send, nrec);
      W.consumed = start ? q : r0;
      W.kept = start ? nf + t : f0;
      W.nr = nrec;
      if (tf < n_hdr) {
        W.status = code_f == STOP_FRAG ? CRK_E_FRAG
                 : code_f == STOP_INCOMPLETE ? CRK_INCOMPLETE
                 : (nrec > 0 ? CRK_INCOMPLETE : CRK_E_CAPACITY);
      } else {
        W.status = (start && q == E.R.tail) ? CRK_OK : CRK_INCOMPLETE;
      }
      W.stop = true;
      return false;
    }
    // the last accepted header advances the state and the predictors
    SCAN_TRACE(lane == 0, 1, n_hdr);
    const uint32_t t = n_hdr - 1;
    at(t, q, len, last, start, send, nrec);
    W.p = q + 4 + len;
    W.nf = nf + n_hdr;
    if (last) {
      W.nr = nrec + 1;
      W.r0 = W.p;
      W.sum = 0;
      W.f0 = nf + n_hdr;
    } else {
      W.nr = nrec;
      W.sum = send;
      W.r0 = start ? q : r0;
      W.f0 = start ? nf + t : f0;
    }
    if (tstar < kWTT) {
      if (start && last) W.hp1 = hstar;
      else if (!last) W.hp0 = hstar;
    }
    if (tstar == kWTT) return true;
    miss = n_hdr <= 2 ? miss + 1 : 0;
  }
}

// One ring's whole scan by the calling CTA (blockDim.x threads, a multiple of 64): fragment and record
// tables in the ring's index slice, and the ring's result (status, records, kept fragments, consumed).
// S is the CTA's shared walk state.  Used by the K1 kernel (one CTA per ring) and by the persistent
// server (one CTA, rings in turn).
__device__ void scan_ring_cta(const IndexDev& ix, const RingDesc& R, bool bad_window, uint32_t ring,
                              const ConfigDev& cfg, ScanState& S) {
  const uint32_t T = blockDim.x >> 1;                  // threads per group
  const uint32_t grp = threadIdx.x >= T, u = threadIdx.x - grp * T;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5, wpg = nw >> 1;
  const uint32_t FC = ix.frags_per_ring, RC = ix.recs_per_ring;
  const uint64_t fbase = (uint64_t)ring * FC, rbase = (uint64_t)ring * RC;
  if (threadIdx.x == 0) {
    ix.rings[ring] = R;
    S.p = S.r0 = R.head;
    S.sum = 0;
    S.f0 = S.nf = S.nr = 0;
    S.hp[0] = cfg.guess & 0x7fffffffu;
    S.hp[1] = kNoPred;
    S.done = bad_window;
    S.wide = 0;
    S.status = CRK_E_ARG;
    S.consumed = R.head;
    S.kept_frags = 0;
  }
  cta_barrier();
  const Env E{ix, R, cfg.max_record_bytes, fbase, rbase, FC, RC};
  for (;;) {
    const bool done = S.done, wide_mode = S.wide;
    cta_barrier();  // everyone has read the mode before warp 0 / the round changes S
    if (done) break;
    if (!wide_mode) {
      // warp rounds / chase passes in warp 0 until a stop or a long regular run; the others wait
      if (warp == 0) {
        Walk W{S.p, S.r0, S.sum, S.nf, S.nr, S.f0, S.hp[0], S.hp[1], false, 0, 0, 0};
        const bool wide = warp_rounds(E, W, lane);
        __syncwarp();
        if (lane == 0) {
          if (W.stop) {
            S.consumed = W.consumed;
            S.kept_frags = W.kept;
            S.nr = W.nr;
            S.status = W.status;
            S.done = 1;
          } else {
            S.p = W.p;
            S.r0 = W.r0;
            S.sum = W.sum;
            S.nf = W.nf;
            S.nr = W.nr;
            S.f0 = W.f0;
            S.hp[0] = W.hp0;
            S.hp[1] = W.hp1;
            S.wide = wide;
          }
        }
      }
      cta_barrier();
      continue;
    }
    const uint64_t p = S.p, r0 = S.r0, sum = S.sum;
    const uint32_t nf = S.nf, nr = S.nr, f0 = S.f0;
    // ---- both groups speculate from the true header at p; thread u owns candidates u + j*T
    // both predictors are read here, before the round's first barrier: the thread that advances the
    // walk rewrites S.hp at the end of this round, possibly while others are still past that barrier
    const uint32_t hp0 = S.hp[0], hp1 = S.hp[1];
    uint32_t hpred = grp ? hp1 : hp0;
    const uint64_t stride = 4 + (uint64_t)(hpred & 0x7fffffffu);
    // a round uses kJ candidates per thread only after a round that accepted every candidate (a long
    // regular run: big records); otherwise one, which keeps the round short
    const uint32_t jn = S.wide ? kJ : 1u, TT = T * jn;
    uint32_t hv[kJ], w0[kJ], w1[kJ];
    bool vv[kJ];
    uint32_t first_bad = TT;
    // all candidate loads are issued before any is used: each header is read as the two aligned words
    // that contain it (branch-free, any alignment, across the wrap) and joined by a funnel shift
#pragma unroll
    for (uint32_t j = 0; j < kJ; ++j) {
      const uint64_t q = p + (uint64_t)(u + j * T) * stride;
      vv[j] = j < jn && q + 4 <= R.tail;
      const uint64_t a = q & ~3ull;
      w0[j] = vv[j] ? CRK_RO_LD(reinterpret_cast<const uint32_t*>(R.base + (a & R.mask))) : 0u;
      w1[j] = (vv[j] && (q & 3)) ? CRK_RO_LD(reinterpret_cast<const uint32_t*>(R.base + ((a + 4) & R.mask))) : 0u;
    }
    uint32_t bh = 0, bv = 0;  // header and validity of this thread's first mismatching candidate
#pragma unroll
    for (uint32_t j = 0; j < kJ; ++j) {
      const uint32_t t = u + j * T;
      const uint64_t q = p + (uint64_t)t * stride;
      hv[j] = bswap32(__funnelshift_r(w0[j], w1[j], 8 * (uint32_t)(q & 3)));
      if (j < jn && first_bad == TT && !(vv[j] && hv[j] == hpred)) { first_bad = t; bh = hv[j]; bv = vv[j]; }
    }
    // per-group first mismatch (groups are whole warps); the warp publishes the mismatching header too
    const uint32_t wm = __reduce_min_sync(0xffffffffu, first_bad);
    const uint32_t own = __ffs(__ballot_sync(0xffffffffu, first_bad == wm)) - 1;
    const uint32_t oh = __shfl_sync(0xffffffffu, bh, own), ov = __shfl_sync(0xffffffffu, bv, own);
    if (lane == 0) { S.gmin[warp] = wm; S.gh[warp] = oh; S.gv[warp] = ov; }
    cta_barrier();
    uint32_t ts0 = TT, ts1 = TT, ws0 = 0, ws1 = 0;
    for (uint32_t w = 0; w < nw; ++w) {
      const uint32_t g = S.gmin[w];
      if (w < wpg) { if (g < ts0) { ts0 = g; ws0 = w; } }
      else if (g < ts1) { ts1 = g; ws1 = w; }
    }
    // the group with the longer verified run wins (ties: group 0)
    const uint32_t win = ts1 > ts0;
    const uint32_t tstar = win ? ts1 : ts0;
    const uint32_t wstar = win ? ws1 : ws0;
    const bool mine = grp == win;
    hpred = win ? hp1 : hp0;
    const uint64_t Lp = hpred & 0x7fffffffu;
    const uint64_t wstride = 4 + Lp;  // the winning predictor's stride (stride is this group's own)
    const uint32_t lastp = hpred >> 31;
    const bool end_at_star = tstar < TT && !S.gv[wstar];
    const uint32_t n_hdr = tstar == TT ? TT : (end_at_star ? tstar : tstar + 1);
    const uint32_t hstar = S.gh[wstar];

    // per-header closed forms (headers 0..tstar-1 equal hpred); checks in the oracle's order.  The checks
    // are monotone along the run (a record's running length, the end of header t's data and the fragment
    // / record counts only grow; with lastp every header 1..u*-1 is a whole record of length Lp), so
    // headers 0, 1 and n_hdr - 1 passing means all pass, and the per-candidate search for the first
    // failure (one more barrier) is skipped.
    bool any_fail = false;
    for (uint32_t k = 0; k < 3; ++k) {
      const uint32_t t = k == 0 ? 0u : (k == 1 ? (n_hdr > 1 ? 1u : 0u) : (n_hdr ? n_hdr - 1 : 0u));
      if (t >= n_hdr) continue;
      const uint64_t q = p + (uint64_t)t * wstride;
      const uint64_t len = (t < tstar) ? Lp : (uint64_t)(hstar & 0x7fffffffu);
      const bool start = (t == 0) ? (p == r0) : (lastp != 0);
      uint64_t send;
      if (!lastp) send = sum + (uint64_t)t * Lp + len;
      else send = (t == 0) ? (start ? len : sum + len) : len;
      const uint32_t nrec = lastp ? nr + t : nr;
      any_fail |= send > cfg.max_record_bytes || q + 4 + len > R.tail || nf + t >= FC || (start && nrec >= RC);
    }
    uint32_t tf = 0xffffffffu, code_f = STOP_NONE;
    if (any_fail) {
      uint32_t codes[kJ];
      uint32_t first_fail = 0xffffffffu;
#pragma unroll
      for (uint32_t j = 0; j < kJ; ++j) {
        const uint32_t t = u + j * T;
        const uint64_t q = p + (uint64_t)t * wstride;
        const uint64_t len = (t < tstar) ? Lp : (uint64_t)(hstar & 0x7fffffffu);
        const bool start = (t == 0) ? (p == r0) : (lastp != 0);
        uint64_t send;  // logical end of header t within its record (segmented prefix sum of lengths)
        if (!lastp) send = sum + (uint64_t)t * Lp + len;
        else send = (t == 0) ? (start ? len : sum + len) : len;
        const uint32_t nrec = lastp ? nr + t : nr;  // completed records before header t
        uint32_t code = STOP_NONE;
        if (mine && j < jn && t < n_hdr) {
          if (send > cfg.max_record_bytes) code = STOP_FRAG;
          else if (q + 4 + len > R.tail) code = STOP_INCOMPLETE;
          else if (nf + t >= FC || (start && nrec >= RC)) code = STOP_CAP;
        }
        codes[j] = code;
        if (code != STOP_NONE && first_fail == 0xffffffffu) first_fail = t;
      }
      uint32_t my_code = STOP_NONE;
#pragma unroll
      for (uint32_t j = 0; j < kJ; ++j)
        if (u + j * T == first_fail) my_code = codes[j];
      const uint32_t fm = __reduce_min_sync(0xffffffffu, first_fail);
      const uint32_t fown = __ffs(__ballot_sync(0xffffffffu, first_fail == fm)) - 1;
      const uint32_t fc = __shfl_sync(0xffffffffu, my_code, fown);
      if (lane == 0) { S.fmin[warp] = fm; S.fcode[warp] = fc; }
      cta_barrier();
      for (uint32_t w = 0; w < nw; ++w)
        if (S.fmin[w] < tf) { tf = S.fmin[w]; code_f = S.fcode[w]; }
    }
    const uint32_t n_emit = tf < n_hdr ? tf : n_hdr;

#pragma unroll
    for (uint32_t j = 0; j < kJ; ++j) {
      const uint32_t t = u + j * T;
      if (!mine || j >= jn) break;
      const uint64_t q = p + (uint64_t)t * wstride;
      const uint64_t len = (t < tstar) ? Lp : (uint64_t)(hstar & 0x7fffffffu);
      const uint32_t last = (t < tstar) ? lastp : (hstar >> 31);
      const bool start = (t == 0) ? (p == r0) : (lastp != 0);
      uint64_t send;
      if (!lastp) send = sum + (uint64_t)t * Lp + len;
      else send = (t == 0) ? (start ? len : sum + len) : len;
      const uint32_t nrec = lastp ? nr + t : nr;
      // emit fragments (and the records they complete)
      if (t < n_emit) {
        const uint64_t fs = fbase + nf + t;
        ix.frag_phys[fs] = q + 4;
        ix.frag_lstart[fs] = send - len;
        ix.frag_hdr[fs] = (uint32_t)len | (last << 31);
        if (last) {
          const uint64_t rs = rbase + nrec;
          ix.rec_begin[rs] = start ? q : r0;
          ix.rec_len[rs] = send;
          ix.rec_frag0[rs] = (uint32_t)(fbase + (start ? nf + t : f0));
          ix.rec_nfrags[rs] = start ? 1u : nf + t - f0 + 1;
        }
      }
      // the stopping candidate (failure at tf, or no readable header at tstar) records the outcome
      const bool stops_here = (tf < n_hdr) ? (t == tf) : (end_at_star && t == tstar);
      if (stops_here) {
        S.consumed = start ? q : r0;
        S.kept_frags = start ? nf + t : f0;
        S.nr = nrec;
        if (tf < n_hdr) {
          const uint32_t c = code_f;
          S.status = c == STOP_FRAG ? CRK_E_FRAG
                   : c == STOP_INCOMPLETE ? CRK_INCOMPLETE
                   : (nrec > 0 ? CRK_INCOMPLETE : CRK_E_CAPACITY);
        } else {
          S.status = (start && q == R.tail) ? CRK_OK : CRK_INCOMPLETE;
        }
        S.done = 1;
      }
      // the last accepted header advances the state and the predictors
      if (!stops_here && tf >= n_hdr && !end_at_star && t == n_hdr - 1) {
        S.wide = tstar == TT;
        SCAN_TRACE(true, 3, n_hdr);
        S.p = q + 4 + len;
        S.nf = nf + n_hdr;
        if (last) {
          S.nr = nrec + 1;
          S.r0 = q + 4 + len;
          S.sum = 0;
          S.f0 = nf + n_hdr;
        } else {
          S.nr = nrec;
          S.sum = send;
          S.r0 = start ? q : r0;
          S.f0 = start ? nf + t : f0;
        }
        if (tstar < TT) {
          // a single-fragment record's shape becomes predictor 1; a non-last fragment of another length
          // becomes predictor 0 (a new stride); the last fragment of a multi-fragment record changes nothing
          if (start && last) S.hp[1] = hstar;
          else if (!last) S.hp[0] = hstar;
        }
      }
    }
    cta_barrier();
  }
  SCAN_TRACE(threadIdx.x == 0, 0, 0);  // end marker
  if (threadIdx.x == 0) {
    crk_ring_result& rr = ix.res[ring];
    rr.status = S.status;
    rr.n_records = S.nr;
    rr.n_frags = S.kept_frags;
    rr.consumed = S.consumed;
    rr.reply_bytes = 0;
  }
  cta_barrier();
}

// Dense record numbering = exclusive prefix of the rings' record counts (one thread).
__device__ __forceinline__ void dense_numbering(const IndexDev& ix, uint32_t n_rings) {
  uint32_t acc = 0;
  for (uint32_t r = 0; r < n_rings; ++r) {
    volatile crk_ring_result* vr = ix.res + r;
    ix.rec_prefix[r] = acc;
    vr->rec_base = acc;
    acc += vr->n_records;
  }
  ix.rec_prefix[n_rings] = acc;
  *ix.total = acc;
}

// The same numbering when one CTA scanned every ring: after ring r's scan_ring_cta, thread 0 sets
// prefix[r + 1] = prefix[r] + S.nr (shared memory), so no result is read back; thread 0 then writes the
// tables with stores only.
__device__ __forceinline__ void dense_numbering_cta(const IndexDev& ix, uint32_t n_rings, const uint32_t* prefix) {
  for (uint32_t r = 0; r < n_rings; ++r) {
    ix.rec_prefix[r] = prefix[r];
    ix.res[r].rec_base = prefix[r];
  }
  ix.rec_prefix[n_rings] = prefix[n_rings];
  *ix.total = prefix[n_rings];
}

}  // namespace
}  // namespace crk
