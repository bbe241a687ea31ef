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
#include "crk_device.cuh"

namespace crk {

namespace {

enum : uint32_t { STOP_NONE = 0, STOP_FRAG = 1, STOP_INCOMPLETE = 2, STOP_CAP = 3 };
constexpr uint32_t kNoPred = 0xffffffffu;  // a predictor value no header is expected to match
constexpr uint32_t kJ = 4;                 // candidate headers per thread and round (independent loads)

struct ScanState {
  uint64_t p, r0, sum;
  uint32_t f0, nf, nr;
  uint32_t hp[2];
  uint32_t done;
  int32_t status;
  uint64_t consumed;
  uint32_t kept_frags;
  uint32_t wide;
  uint32_t gmin[32], gh[32], gv[32];  // per warp: first mismatch, its header, its validity
  uint32_t fmin[32], fcode[32];       // per warp: first failing check and its code
};

__global__ void __launch_bounds__(1024) frame_scan_kernel(IndexDev ix, ScanRingsParam P, ConfigDev cfg) {
  const uint32_t ring = blockIdx.x;
  RingDesc R = P.r[ring];
  bool bad_window = false;
  if (P.doorbell) {  // cursors published by the host at execution time
    R.head = P.doorbell[ring];
    R.tail = P.doorbell[P.n_rings + ring];
    bad_window = R.tail < R.head || R.tail - R.head > R.mask + 1;
    if (bad_window) R.tail = R.head;
  }
  const uint32_t T = blockDim.x >> 1;                  // threads per group
  const uint32_t grp = threadIdx.x >= T, u = threadIdx.x - grp * T;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5, wpg = nw >> 1;
  const uint32_t FC = ix.frags_per_ring, RC = ix.recs_per_ring;
  const uint64_t fbase = (uint64_t)ring * FC, rbase = (uint64_t)ring * RC;
  __shared__ ScanState S;
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
  __syncthreads();
  while (!S.done) {
    const uint64_t p = S.p, r0 = S.r0, sum = S.sum;
    const uint32_t nf = S.nf, nr = S.nr, f0 = S.f0;
    // ---- both groups speculate from the true header at p; thread u owns candidates u + j*T
    uint32_t hpred = S.hp[grp];
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
      w0[j] = vv[j] ? __ldg(reinterpret_cast<const uint32_t*>(R.base + (a & R.mask))) : 0u;
      w1[j] = vv[j] ? __ldg(reinterpret_cast<const uint32_t*>(R.base + ((a + 4) & R.mask))) : 0u;
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
    __syncthreads();
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
    hpred = S.hp[win];
    const uint64_t Lp = hpred & 0x7fffffffu;
    const uint32_t lastp = hpred >> 31;
    const bool end_at_star = tstar < TT && !S.gv[wstar];
    const uint32_t n_hdr = tstar == TT ? TT : (end_at_star ? tstar : tstar + 1);
    const uint32_t hstar = S.gh[wstar];

    // per-header closed forms (headers 0..tstar-1 equal hpred); checks in the oracle's order
    uint32_t codes[kJ];
    uint32_t first_fail = 0xffffffffu;
#pragma unroll
    for (uint32_t j = 0; j < kJ; ++j) {
      const uint32_t t = u + j * T;
      const uint64_t q = p + (uint64_t)t * stride;
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
    __syncthreads();
    uint32_t tf = 0xffffffffu, code_f = STOP_NONE;
    for (uint32_t w = 0; w < nw; ++w)
      if (S.fmin[w] < tf) { tf = S.fmin[w]; code_f = S.fcode[w]; }
    const uint32_t n_emit = tf < n_hdr ? tf : n_hdr;

#pragma unroll
    for (uint32_t j = 0; j < kJ; ++j) {
      const uint32_t t = u + j * T;
      if (!mine || j >= jn) break;
      const uint64_t q = p + (uint64_t)t * stride;
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
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    crk_ring_result& rr = ix.res[ring];
    rr.status = S.status;
    rr.n_records = S.nr;
    rr.n_frags = S.kept_frags;
    rr.consumed = S.consumed;
    rr.reply_bytes = 0;
    __threadfence();
    const uint32_t done = atomicAdd(ix.ticket, 1u);
    if (done == gridDim.x - 1) {
      // last ring: dense record numbering = exclusive prefix over rings
      __threadfence();
      uint32_t acc = 0;
      for (uint32_t r = 0; r < gridDim.x; ++r) {
        volatile crk_ring_result* vr = ix.res + r;
        ix.rec_prefix[r] = acc;
        vr->rec_base = acc;
        acc += vr->n_records;
      }
      ix.rec_prefix[gridDim.x] = acc;
      *ix.total = acc;
      *ix.ticket = 0;
    }
  }
}

}  // namespace

cudaError_t launch_frame_scan(const IndexDev& ix, const ScanRingsParam& p, const ConfigDev& cfg, cudaStream_t s) {
  prof_mark(PROF_SCAN, true, s);
  frame_scan_kernel<<<p.n_rings, cfg.scan_threads, 0, s>>>(ix, p, cfg);
  count_launch();
  prof_mark(PROF_SCAN, false, s);
  return cudaGetLastError();
}

}  // namespace crk
