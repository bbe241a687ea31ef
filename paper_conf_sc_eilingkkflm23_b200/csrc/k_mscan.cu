// K1 for long windows: the chunked, multi-CTA record-marking scan (RFC 5531 §11; SURVEY.md §7 "Hard parts":
// a chained scan across CTAs carrying next header position, header count and record id).
//
// The header chain is sequential: header k+1 sits at p[k] + 4 + len[k].  One CTA per ring walking it pays one
// memory round trip per speculative round (~1 record per round for mixed streams, one hop per round for
// irregular framing: PAPER.md:98 needs fragmented records for large parameters).  Here a ring window is cut
// into chunks of S bytes, one CTA each, and every chunk is walked at once:
//
//  K1a (chunk_walk_kernel), CTA = chunk i of ring r, covering cursors [c_i, c_{i+1}):
//   * Chunk 0 starts at the window head, a true header.  Any other chunk does not know where its first header
//     is, but it is close: the last header before c_i carries at most kLmax bytes (greedy F = 64 KiB framing,
//     and C4's irregular fragments are <= 64 KiB), so the entry x_i lies in the landing zone
//     [c_i, c_i + kLmax + 4).  The zone is staged into shared memory with one TMA bulk copy, and every byte
//     position in it is tested as a header: a candidate's length must be <= kLmax, then the chain from it is
//     followed until it is well past the zone (zone bytes from shared memory, the rest from the ring).  In
//     random payload bytes a false candidate survives a hop with probability ~2^-15, a true header always;
//     candidates on another candidate's chain are dropped, and the kCand best distinct chains (alive first,
//     then lowest position) are kept.
//   * One warp per candidate walks its chain up to c_{i+1} with the speculative rounds of the one-CTA scan
//     (two predictor groups; a round accepts every header up to the first mismatch, which is itself true)
//     and logs each header (cursor, raw header) -- no checks yet: they depend on the state at the chunk's
//     true entry.  A summary of the log (count, last-fragment count and position, length sums, exit cursor)
//     is all the next step needs.
//   * The last CTA of the ring to finish (ticket) resolves it: the true chain enters chunk 0 at the head and
//     enters chunk i+1 at the exit of the candidate chain whose start equals chunk i's entry.  Each chunk is a
//     map candidate -> candidate of the next chunk (or end of chain / no match); an exclusive block scan of
//     map composition gives every chunk's true candidate at once, a scan of (fragment, record) counts gives
//     the fragment and record numbers at each chunk's entry, and a segmented scan gives the record being
//     built there (its start, its logical length so far, its first fragment).  When a chunk's entry is no
//     candidate's start (a fragment longer than kLmax crossed the boundary, payload bytes that look like a
//     chain, a log that overflowed) the ring falls back to the one-CTA scan: correct, just not faster.
//  K1b (chunk_emit_kernel), CTA = chunk: the true chain's log is turned into index entries by take_hops
//   (k_scan.cuh) -- the same closed forms and checks in or_frame_scan's order the one-CTA scan uses -- from
//   the chunk's entry state.  A failing check records its outcome; the first failing hop of the ring (lowest
//   fragment number, atomicMin) decides the ring's result, else the end of the chain does.  The last CTA
//   numbers the records densely across rings.
//
// Every step is exact (no speculation survives unverified): a candidate is used only when the previous
// chunk's true chain exits exactly at its start.  Rings whose window is short stay on the one-CTA scan
// (scan_ring_cta), inside the same launches.
#include <mutex>

#include "k_scan.cuh"

namespace crk {

namespace {

enum : uint32_t { CH_NONE = 0, CH_EXIT = 1, CH_END_WINDOW = 2, CH_END_DATA = 3, CH_OVERFLOW = 4 };
constexpr uint32_t kLmax = 65536;              // longest fragment a landing zone is sized for
constexpr uint32_t kZone = kLmax + 4;          // entry positions c_i .. c_i + kZone - 1
constexpr uint32_t kZoneBytes = 65536 + 64;    // staged: 16-byte alignment slack + zone + the last header
constexpr uint32_t kSurv = 1024;               // zone positions kept after the first hop
constexpr uint32_t kThreads = 256;
constexpr uint32_t kMaxRingChunks = kThreads;  // the resolver holds one chunk per thread
static_assert(kMaxRingChunks * kCand * sizeof(ChainSum) <= kZoneBytes, "a ring's chain summaries fit the zone");
constexpr uint32_t kWJ4 = 4;                   // candidate headers per lane and walk round (64 per group)
constexpr uint32_t kWT = 16 * kWJ4;

#ifdef CRK_MSCAN_TRACE
// Diagnostic build only (build.py build_variant("mtrace", ["CRK_MSCAN_TRACE"])): per K1a CTA, %globaltimer at
// its start and after each phase (zone staged, first hop, scoring, selection, walk, resolve).
constexpr uint32_t kTraceCtas = 4096, kTracePh = 12;
__device__ unsigned long long g_mtrace[kTraceCtas][kTracePh];
__device__ __forceinline__ void mtrace(uint32_t ph) {
  if (threadIdx.x == 0 && blockIdx.x < kTraceCtas) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    g_mtrace[blockIdx.x][ph] = t;
  }
}
#define MTRACE(ph) mtrace(ph)
#else
#define MTRACE(ph) do { } while (0)
#endif

constexpr uint32_t kInlineChunks = 32;  // rings of at most this many chunks are emitted by their resolving CTA

struct ChunkParam {
  uint32_t n_rings;
  uint32_t need_emit;              // some ring has more than kInlineChunks chunks: chunk_emit_kernel runs
  uint32_t chunk0[kMaxRings + 1];  // exclusive prefix of the rings' chunk counts
  uint64_t S[kMaxRings];           // chunk size per ring
  RingDesc r[kMaxRings];
};

__device__ __forceinline__ void locate(const ChunkParam& P, uint32_t g, uint32_t& r, uint32_t& i, uint32_t& K) {
  uint32_t lo = 0;
  while (lo + 1 < P.n_rings && P.chunk0[lo + 1] <= g) ++lo;
  r = lo;
  i = g - P.chunk0[lo];
  K = P.chunk0[lo + 1] - P.chunk0[lo];
}

// Coherent (L2) loads of what other CTAs of the same launch wrote.
__device__ __forceinline__ ChainSum ld_sum(const ChainSum* p) {
  ChainSum s;
  const uint4* q = reinterpret_cast<const uint4*>(p);
  uint4* d = reinterpret_cast<uint4*>(&s);
  d[0] = __ldcg(q);
  d[1] = __ldcg(q + 1);
  d[2] = __ldcg(q + 2);
  d[3] = __ldcg(q + 3);
  return s;
}

// Header at cursor q from the staged zone (bytes of cursor a0 onward) when it lies there, else from the ring.
__device__ __forceinline__ uint32_t hdr_at(const RingDesc& R, const uint8_t* zone, uint64_t a0, uint64_t q) {
  const uint64_t o = q - a0;
  if (q >= a0 && o + 8 <= kZoneBytes) {
    const uint32_t* w = reinterpret_cast<const uint32_t*>(zone + (o & ~3ull));
    return join_hdr(q, w[0], w[1]);
  }
  uint32_t w0, w1;
  load_hdr(R, q, true, w0, w1);
  return join_hdr(q, w0, w1);
}

struct SelSmem {
  uint64_t bar;
  uint32_t nsurv;
  uint32_t surv[kSurv];
  uint32_t key[kSurv];
  uint32_t red[32];
  uint32_t reached[(kZone + 31) / 32];  // zone positions some survivor's chain passes through
};

// The landing zone of chunk i >= 1: up to kCand candidate entries, best first (written to cand[]).
// A true header's chain runs on to the chunk's end with every length <= kLmax; a chain started inside payload
// bytes or inside a CALL header's zero words (AUTH_NONE cred / verf, small pointers) soon reads an implausible
// length and dies.  Survivors of the first hop are followed until they are kFar bytes past the chunk start
// (or reach the window's end, or kHops hops): the ones still alive rank first.  A survivor another survivor's
// chain passes through is not a root -- its chain is the other's suffix, e.g. the true headers after the
// entry -- and ranks after the roots, so the kCand slots go to distinct chains first: the true entry, and at
// most a few false starts that merge into the true chain or look like one.  (The entry itself is a non-root
// only when a false start's chain runs into it; it is then the first non-root.)  Ties: lowest position.
constexpr uint32_t kHops = 64;
constexpr uint64_t kFar = 2ull * kZone;
__device__ uint32_t select_candidates(const RingDesc& R, uint64_t ci, uint64_t cn, uint8_t* zone, SelSmem& M,
                                      uint64_t* cand) {
  const uint64_t a0 = ci & ~15ull;
  const uint32_t zoff = (uint32_t)(ci - a0);
  uint64_t zl = kZone;  // positions u: q = ci + u < cn, q + 4 <= tail
  if (cn - ci < zl) zl = cn - ci;
  const uint64_t lim = R.tail >= ci + 4 ? R.tail - ci - 3 : 0;
  if (lim < zl) zl = lim;
  const uint64_t far = ci + kFar < cn ? ci + kFar : cn;
  if (threadIdx.x == 0) {
    mbar_init(&M.bar, 1);
    M.nsurv = 0;
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  for (uint32_t k = threadIdx.x; k < (kZone + 31) / 32; k += blockDim.x) M.reached[k] = 0;
  __syncthreads();
  if (threadIdx.x == 0) {  // one TMA bulk copy (two across the ring's wrap) of the zone into shared memory
    const uint64_t o = a0 & R.mask, room = R.mask + 1 - o;
    const uint32_t n1 = room < kZoneBytes ? (uint32_t)room : kZoneBytes;
    mbar_arrive_expect_tx(&M.bar, kZoneBytes);
    bulk_g2s(zone, R.base + o, n1, &M.bar);
    if (n1 < kZoneBytes) bulk_g2s(zone + n1, R.base, kZoneBytes - n1, &M.bar);
  }
  mbar_wait(&M.bar, 0);
  MTRACE(1);
  // hop 1 at every position: aligned word k of the zone holds the first bytes of the headers at 4k .. 4k+3
  const uint32_t* zw = reinterpret_cast<const uint32_t*>(zone);
  const uint32_t nwords = (uint32_t)((zoff + zl + 3) / 4);
  // A header's length is <= kLmax = 0x10000 only if its first two bytes satisfy (b0 & 0x7f) = 0 and
  // (b1 & 0xfe) = 0, i.e. the little-endian 16-bit lane b0 | b1 << 8 masked with 0xfe7f is zero.  Each thread
  // takes 16 zone bytes per step (LDS.128 + the next word): the even-offset pairs are the 16-bit lanes of each
  // word, the odd ones those of the word shifted by a byte, and a lane-wise "has a zero lane" test (no
  // branches) flags the rare words that get the exact per-position test.  Random payload flags a position
  // with probability 2^-14.
  const uint32_t nchunks = (nwords + 3) / 4;
  const uint4* zv = reinterpret_cast<const uint4*>(zone);
  for (uint32_t c = threadIdx.x; c < nchunks; c += blockDim.x) {
    const uint4 v = zv[c];
    const uint32_t wv[5] = {v.x, v.y, v.z, v.w, zw[4 * c + 4]};
    uint32_t flag = 0;
#pragma unroll
    for (uint32_t q = 0; q < 4; ++q) {
      const uint32_t e = wv[q] & 0xfe7ffe7fu, o = __funnelshift_r(wv[q], wv[q + 1], 8) & 0xfe7ffe7fu;
      const uint32_t ze = (e - 0x00010001u) & ~e & 0x80008000u, zo = (o - 0x00010001u) & ~o & 0x80008000u;
      flag |= (ze | zo) ? 1u << q : 0u;
    }
    while (flag) {
      const uint32_t q = __ffs(flag) - 1;
      flag &= flag - 1;
      const uint32_t k = 4 * c + q;
      if (k >= nwords) break;
      const uint32_t w0 = wv[q], w1 = wv[q + 1];
      for (uint32_t b = 0; b < 4; ++b) {
        const uint32_t h = bswap32(__funnelshift_r(w0, w1, 8 * b));
        const int64_t u = (int64_t)(4 * k + b) - zoff;
        if ((h & 0x7fffffffu) <= kLmax && u >= 0 && (uint64_t)u < zl) {
          const uint32_t s = atomicAdd(&M.nsurv, 1u);
          if (s < kSurv) M.surv[s] = (uint32_t)u;
        }
      }
    }
  }
  __syncthreads();
  MTRACE(2);
  const uint32_t ns = min(M.nsurv, kSurv);
  for (uint32_t s = threadIdx.x; s < ns; s += blockDim.x) {  // follow each survivor's chain
    const uint32_t u = M.surv[s];
    uint64_t p = ci + u;
    bool alive = false;
    for (uint32_t hop = 0; hop < kHops; ++hop) {
      if (p >= far || p + 4 > R.tail) { alive = true; break; }  // far enough, or the end of the window
      if (hop) {
        const uint64_t v = p - ci;
        if (v < zl) atomicOr(&M.reached[v >> 5], 1u << (v & 31));
      }
      const uint32_t len = hdr_at(R, zone, a0, p) & 0x7fffffffu;
      if (len > kLmax) break;
      p += 4 + (uint64_t)len;
      alive = hop + 1 == kHops;
    }
    M.key[s] = ((alive ? 0u : 1u) << 19) | u;  // u < 2^17; bit 18: not a root
  }
  __syncthreads();
  MTRACE(3);
  for (uint32_t s = threadIdx.x; s < ns; s += blockDim.x) {  // survivors on another survivor's chain rank later
    const uint32_t u = M.key[s] & 0x1ffffu;
    if ((M.reached[u >> 5] >> (u & 31)) & 1) M.key[s] |= 1u << 18;
  }
  __syncthreads();
  uint32_t nc = 0;
  if (ns <= 32) {  // the usual case: warp 0 picks the kCand smallest keys with warp reductions
    if (threadIdx.x < 32) {
      uint32_t key = threadIdx.x < ns ? M.key[threadIdx.x] : 0xffffffffu;
      for (; nc < kCand; ++nc) {
        const uint32_t m = __reduce_min_sync(kFull, key);
        if (m == 0xffffffffu) break;
        if (threadIdx.x == 0) cand[nc] = ci + (m & 0x1ffffu);
        if (key == m) key = 0xffffffffu;
      }
      if (threadIdx.x == 0) M.nsurv = nc;
    }
    __syncthreads();
    return M.nsurv;
  }
  for (; nc < kCand; ++nc) {
    uint32_t m = 0xffffffffu;
    for (uint32_t s = threadIdx.x; s < ns; s += blockDim.x) m = min(m, M.key[s]);
    m = block_min_u32(m, M.red);
    if (m == 0xffffffffu) break;
    if (threadIdx.x == 0) cand[nc] = ci + (m & 0x1ffffu);
    for (uint32_t s = threadIdx.x; s < ns; s += blockDim.x)
      if (M.key[s] == m) M.key[s] = 0xffffffffu;
    __syncthreads();
  }
  return nc;
}

// One warp walks the chain from `start` (a true header or a candidate) while its headers start below cn,
// logging (cursor - ci, header) of each, and writes the log's summary.
__device__ void walk_chain(const RingDesc& R, uint64_t start, uint64_t ci, uint64_t cn, uint32_t guess, uint2* log,
                           ChainSum* out, uint32_t lane) {
  const uint32_t grp = lane >> 4, u = lane & 15;
  const uint64_t tail = R.tail;
  uint64_t p = start;
  uint32_t hp0 = guess & 0x7fffffffu, hp1 = kNoPred, n = 0, kind;
  bool prev_last = true;
  for (;;) {
    if (p + 4 > tail) { kind = CH_END_WINDOW; break; }
    if (p >= cn) { kind = CH_EXIT; break; }
    const uint32_t hm = grp ? hp1 : hp0;
    const uint64_t sm = 4 + (uint64_t)(hm & 0x7fffffffu);
    uint32_t w0[kWJ4], w1[kWJ4];
    bool vv[kWJ4];
#pragma unroll
    for (uint32_t j = 0; j < kWJ4; ++j) {
      const uint64_t q = p + (uint64_t)(u + 16 * j) * sm;
      vv[j] = q < cn && q + 4 <= tail;
      load_hdr(R, q, vv[j], w0[j], w1[j]);
    }
    uint32_t first_bad = kWT, bh = 0, bv = 0;
#pragma unroll
    for (uint32_t j = 0; j < kWJ4; ++j) {
      const uint32_t t = u + 16 * j;
      const uint32_t h = join_hdr(p + (uint64_t)t * sm, w0[j], w1[j]);
      if (first_bad == kWT && !(vv[j] && h == hm)) { first_bad = t; bh = h; bv = vv[j]; }
    }
    const uint32_t ts0 = __reduce_min_sync(kFull, grp == 0 ? first_bad : kWT);
    const uint32_t ts1 = __reduce_min_sync(kFull, grp == 1 ? first_bad : kWT);
    const uint32_t win = ts1 > ts0, tstar = win ? ts1 : ts0;
    uint32_t hstar = 0, vstar = 0;
    if (tstar < kWT) {
      const uint32_t own = __ffs(__ballot_sync(kFull, grp == win && first_bad == tstar)) - 1;
      hstar = __shfl_sync(kFull, bh, own);
      vstar = __shfl_sync(kFull, bv, own);
    }
    const uint32_t hp = win ? hp1 : hp0;
    const uint64_t Lp = hp & 0x7fffffffu, stride = 4 + Lp;
    const uint32_t lastp = hp >> 31;
    // headers 0 .. tstar-1 equal hp (exact positions by induction); header tstar is true when readable
    const bool star_in = tstar < kWT && vstar;
    uint32_t n_ok = star_in ? tstar + 1 : tstar;
    bool end_data = false;  // the first accepted header whose data runs past the window's tail ends the chain
    if (tstar > 0 && p + 4 + Lp > tail) {
      n_ok = 1;
      end_data = true;
    } else if (tstar > 0) {
      const uint64_t td = (tail - 4 - Lp - p) / stride + 1;  // first t < tstar with data past tail
      if (td < tstar) { n_ok = (uint32_t)td + 1; end_data = true; }
    }
    if (!end_data && star_in && p + (uint64_t)tstar * stride + 4 + (hstar & 0x7fffffffu) > tail) end_data = true;
    if (n + n_ok > kLogCap) { kind = CH_OVERFLOW; break; }
    for (uint32_t t = lane; t < n_ok; t += 32)
      log[n + t] = make_uint2((uint32_t)(p + (uint64_t)t * stride - ci), t < tstar ? hp : hstar);
    n += n_ok;
    if (end_data) { kind = CH_END_DATA; break; }
    if (star_in) {
      const uint64_t qs = p + (uint64_t)tstar * stride;
      const bool st = tstar == 0 ? prev_last : lastp != 0;
      const uint32_t ls = hstar >> 31;
      if (st && ls) hp1 = hstar;
      else if (!ls) hp0 = hstar;
      prev_last = ls;
      p = qs + 4 + (hstar & 0x7fffffffu);
    } else {
      p += (uint64_t)tstar * stride;  // the next header position, not readable in this chunk
      prev_last = lastp;
    }
  }
  __syncwarp();
  // summary of the log: sums of lengths, last fragments, the record state after the last one
  uint64_t sum_total = 0, sum_after = 0, r0_after = 0;
  uint32_t nlast = 0;
  int32_t idx_last = -1;
  for (uint32_t k0 = 0; k0 < n; k0 += 32) {
    const bool v = k0 + lane < n;
    const uint2 e = v ? log[k0 + lane] : make_uint2(0, 0);
    const uint64_t len = v ? (uint64_t)(e.y & 0x7fffffffu) : 0;
    const uint32_t lm = __ballot_sync(kFull, v && (e.y >> 31));
    uint64_t s = len, sa = 0;
    if (lm) {
      const uint32_t L = 31 - __clz(lm);
      sa = lane > L ? len : 0;
      const uint64_t eL = __shfl_sync(kFull, (uint64_t)e.x + 4 + len, L);
      r0_after = ci + eL;
      idx_last = (int32_t)(k0 + L);
    } else {
      sa = len;
    }
#pragma unroll
    for (uint32_t o = 16; o; o >>= 1) {
      s += __shfl_xor_sync(kFull, s, o);
      sa += __shfl_xor_sync(kFull, sa, o);
    }
    sum_total += s;
    sum_after = lm ? sa : sum_after + sa;
    nlast += __popc(lm);
  }
  if (lane == 0) {
    ChainSum c;
    c.start = start;
    c.exit = p;
    c.r0_after = r0_after;
    c.sum_after = sum_after;
    c.sum_total = sum_total;
    c.n = n;
    c.nlast = nlast;
    c.idx_last = idx_last;
    c.kind = kind;
    c.pad_ = 0;
    *out = c;
  }
}

// ---- block scans for the resolver (kThreads threads, one chunk each)
template <class T>
__device__ __forceinline__ T shfl_up_t(T v, uint32_t d) {
  static_assert(sizeof(T) % 4 == 0, "32-bit words");
  uint32_t w[sizeof(T) / 4];
  memcpy(w, &v, sizeof(T));
#pragma unroll
  for (uint32_t k = 0; k < sizeof(T) / 4; ++k) w[k] = __shfl_up_sync(kFull, w[k], d);
  memcpy(&v, w, sizeof(T));
  return v;
}

// Exclusive scan in thread order under op(a, b) = "a, then b" (associative, identity id); returns the block
// total.  wsm: 32 T of shared memory.
template <class T, class Op>
__device__ T block_scan_excl(T& v, T id, Op op, T* wsm) {
  const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  T x = v;
#pragma unroll
  for (uint32_t o = 1; o < 32; o <<= 1) {
    const T y = shfl_up_t(x, o);
    if (lane >= o) x = op(y, x);
  }
  __syncthreads();
  if (lane == 31) wsm[w] = x;
  __syncthreads();
  if (w == 0) {  // warp 0 scans the warp totals: wsm[k] <- prefix of warps < k, wsm[nw] <- total
    T t = lane < nw ? wsm[lane] : id, y = t;
#pragma unroll
    for (uint32_t o = 1; o < 32; o <<= 1) {
      const T z = shfl_up_t(y, o);
      if (lane >= o) y = op(z, y);
    }
    T ye = shfl_up_t(y, 1);
    if (lane == 0) ye = id;
    __syncwarp();
    if (lane < nw) wsm[lane] = ye;
    if (lane == nw - 1) wsm[nw] = y;
  }
  __syncthreads();
  const T pre = wsm[w], tot = wsm[nw];
  T xe = shfl_up_t(x, 1);
  if (lane == 0) xe = id;
  v = op(pre, xe);
  return tot;
}

// Candidate maps: byte x of the 8 bytes = where entry x goes; entries 0..3 = the chunk's candidates, 4 = end
// of chain, 5 = no match (6, 7 unused).  Composition is two byte permutes (PRMT) with selectors packed from the
// first map's bytes.
constexpr uint32_t kTerm = 4, kFail = 5;
__device__ __forceinline__ uint32_t sel_of(uint32_t bytes) {  // bytes v0..v3 (each < 8) -> nibbles v0..v3
  const uint32_t t = bytes | (bytes >> 4);
  return __byte_perm(t, 0, 0x4420);
}
struct MapThen {  // (a, then b)[x] = b[a[x]]
  __device__ uint2 operator()(uint2 a, uint2 b) const {
    return make_uint2(__byte_perm(b.x, b.y, sel_of(a.x)), __byte_perm(b.x, b.y, sel_of(a.y)));
  }
};
__device__ __forceinline__ uint2 id_map() { return make_uint2(0x03020100u, 0x07060504u); }
struct AddU2 {
  __device__ uint2 operator()(uint2 a, uint2 b) const { return make_uint2(a.x + b.x, a.y + b.y); }
};
struct Carry {  // the record being built: its start cursor, logical length so far, first fragment
  uint32_t reset, f0;
  uint64_t r0, sum;
};
struct CarryThen {
  __device__ Carry operator()(Carry a, Carry b) const { return b.reset ? b : Carry{a.reset, a.f0, a.r0, a.sum + b.sum}; }
};

struct ResSmem {
  uint64_t bar;
  uint8_t ch[kMaxRingChunks];  // every chunk's true candidate (kTerm / kFail otherwise)
  uint2 wm[32];
  uint2 wc[32];
  Carry wr[32];
  uint32_t fail;
  uint64_t p_end;
  int32_t term;
};

// Where the true chain enters candidate chain j of chunk g (chunk start c): 0 when the chain starts at the
// entry x, k when a false start's chain runs into x at its k-th logged header (k < kMerge), -1 otherwise.  The
// log entries are loaded together (one round trip); an x outside the landing zone is no chunk entry.
constexpr uint32_t kMerge = 16;
__device__ int entry_in_chain(const IndexDev& ix, uint32_t g, uint32_t j, uint64_t c, uint64_t x, const ChainSum& cs) {
  if (cs.start == x) return 0;
  if (cs.start > x || x < c || x - c >= kZone) return -1;
  const uint32_t n = min(cs.n, kMerge);
  const uint2* log = ix.ms.log + ((uint64_t)g * kCand + j) * kLogCap;
  uint32_t o[kMerge];
#pragma unroll
  for (uint32_t k = 1; k < kMerge; ++k) o[k] = k < n ? __ldcg(&log[k].x) : 0xffffffffu;
  const uint32_t xo = (uint32_t)(x - c);
#pragma unroll
  for (uint32_t k = 1; k < kMerge; ++k)
    if (o[k] == xo) return (int)k;
  return -1;
}

// The last chunk CTA of ring r: every chunk's true candidate and entry state (see the file comment).  Thread i
// handles chunk i; every load is a coherent L2 load of what the chunk CTAs wrote (a few round trips in all).
__device__ void resolve_ring(const IndexDev& ix, const ChunkParam& P, uint32_t r, uint32_t K, const RingDesc& R,
                             ResSmem& M, uint8_t* zone) {
  (void)zone;
  const uint32_t g0 = P.chunk0[r];
  const uint32_t i = threadIdx.x;
  const ChainSum* S = ix.ms.sums + (uint64_t)g0 * kCand;  // S[i * kCand + j]
  if (threadIdx.x == 0) {
    M.fail = 0;
    M.term = -1;
    M.p_end = 0;
  }
  MTRACE(7);
  const bool mine = i < K;
  // 1. chunk i's map: candidate j -> the candidate of chunk i + 1 whose chain the exit of j enters
  uint2 f = id_map();
  if (mine) {
    uint64_t ex[kCand], nst[kCand];
    uint32_t kd[kCand];
#pragma unroll
    for (uint32_t j = 0; j < kCand; ++j) {  // this chunk's exits, the next chunk's starts: loaded together
      ex[j] = __ldcg(&S[i * kCand + j].exit);
      kd[j] = __ldcg(&S[i * kCand + j].kind);
      nst[j] = i + 1 < K ? __ldcg(&S[(i + 1) * kCand + j].start) : ~0ull;
    }
    const uint64_t cnext = R.head + (uint64_t)(i + 1) * P.S[r];
    uint32_t m = 0;
#pragma unroll
    for (uint32_t j = 0; j < kCand; ++j) {
      uint32_t to = kFail;
      if (kd[j] == CH_END_WINDOW || kd[j] == CH_END_DATA) {
        to = kTerm;
      } else if (kd[j] == CH_EXIT && i + 1 < K) {
        for (uint32_t jj = 0; jj < kCand && to == kFail; ++jj)
          if (nst[jj] == ex[j]) to = jj;
        for (uint32_t jj = 0; jj < kCand && to == kFail; ++jj)  // a false start that runs into the entry
          if (nst[jj] < ex[j] && ex[j] - cnext < kZone &&
              entry_in_chain(ix, g0 + i + 1, jj, cnext, ex[j], ld_sum(S + (i + 1) * kCand + jj)) > 0)
            to = jj;
      }
      m |= to << (8 * j);
    }
    f = make_uint2(m, 0x07060504u);
  }
  MTRACE(11);
  // 2. chosen_i = (f_{i-1} o ... o f_0)(0): chunk 0's only candidate is the window head
  block_scan_excl(f, id_map(), MapThen(), M.wm);
  MTRACE(8);
  const uint32_t ch = mine ? (f.x & 0xffu) : kTerm;
  if (mine) M.ch[i] = (uint8_t)ch;
  if (ch == kFail) M.fail = 1;
  __syncthreads();
  uint2 cnt = make_uint2(0, 0);
  Carry car{0, 0, 0, 0};
  uint64_t start = 0, exitp = 0;
  uint32_t kind = CH_NONE, skip = 0;
  if (ch < kCand) {
    ChainSum c = ld_sum(S + i * kCand + ch);
    const uint64_t x = i > 0 ? __ldcg(&S[(i - 1) * kCand + M.ch[i - 1]].exit) : c.start;
    if (i > 0) {  // the true entry: the exit of the previous chunk's true chain
      const int sk = entry_in_chain(ix, g0 + i, ch, R.head + (uint64_t)i * P.S[r], x, c);
      if (sk < 0) {
        M.fail = 1;
      } else if (sk > 0) {  // drop the false start's headers before the entry from the summary
        const uint2* log = ix.ms.log + ((uint64_t)(g0 + i) * kCand + ch) * kLogCap;
        uint32_t lasts = 0;
        uint64_t lens = 0;
        for (int e = 0; e < sk; ++e) {
          const uint32_t h = __ldcg(&log[e].y);
          lens += h & 0x7fffffffu;
          lasts += h >> 31;
        }
        c.n -= sk;
        c.nlast -= lasts;
        c.sum_total -= lens;
        if (c.idx_last >= sk) c.idx_last -= sk;
        else { c.idx_last = -1; c.nlast = 0; }
        c.start = x;
        skip = (uint32_t)sk;
      }
    }
    cnt = make_uint2(c.n, c.nlast);
    car = c.nlast ? Carry{1, (uint32_t)c.idx_last + 1, c.r0_after, c.sum_after} : Carry{0, 0, 0, c.sum_total};
    start = c.start;
    exitp = c.exit;
    kind = c.kind;
    if (c.kind == CH_OVERFLOW || c.kind == CH_NONE) M.fail = 1;
  }
  MTRACE(9);
  // 3. fragment / record numbers at each chunk's entry; then the record being built there
  const uint2 tot_cnt = block_scan_excl(cnt, make_uint2(0, 0), AddU2(), M.wc);
  if (car.reset) car.f0 += cnt.x;  // absolute: entry fragment number + index after the last 'last'
  const Carry init{1, 0, R.head, 0};
  const Carry tot_car = block_scan_excl(car, Carry{0, 0, 0, 0}, CarryThen(), M.wr);
  MTRACE(10);
  // 4. entry states
  if (mine) {
    const Carry e = CarryThen()(init, car);
    ChunkState st;
    st.p = start;
    st.r0 = e.r0;
    st.sum = e.sum;
    st.nf = cnt.x;
    st.nr = cnt.y;
    st.f0 = e.f0;
    st.chosen = ch < kCand ? (int32_t)ch : -1;
    st.skip = skip;
    st.pad_ = 0;
    ix.ms.state[g0 + i] = st;
    if (ch < kCand && (kind == CH_END_WINDOW || kind == CH_END_DATA)) {
      M.term = (int32_t)i;
      M.p_end = exitp;
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    RingPlan* pl = ix.ms.plan + r;
    const Carry e = CarryThen()(init, tot_car);
    crk_ring_result rr{};
    const bool at_start = M.p_end == e.r0;  // the window ends where a record would start
    rr.status = (at_start && M.p_end == R.tail) ? CRK_OK : CRK_INCOMPLETE;
    rr.n_records = tot_cnt.y;
    rr.n_frags = at_start ? tot_cnt.x : e.f0;
    rr.consumed = e.r0;
    pl->end = rr;
    pl->fallback = (M.fail || M.term < 0) ? 1u : 0u;
    pl->ticket_a = 0;
    atomicAdd(ix.ms.stats + (pl->fallback ? 1 : 0), 1u);
  }
}

// Emission of chunk g's true chain by one warp (defined below).
__device__ void emit_chunk(const IndexDev& ix, const ChunkParam& P, const ConfigDev& cfg, uint32_t r, uint32_t i,
                           uint32_t g, const RingDesc& R, uint32_t lane);

// Ring r's result from its chunks' emission (the first failing hop, else the end of the chain); resets the
// ring's plan for the next launch.  One thread.
__device__ void finalize_ring(const IndexDev& ix, uint32_t r, bool fb) {
  RingPlan* pl = ix.ms.plan + r;
  if (!fb) {
    const unsigned long long key = __ldcg(&pl->stop_key);
    crk_ring_result rr;
    if (key != ~0ull) {
      const ChunkStop* cs = ix.ms.stops + (key & 0xffffffull);
      rr.status = __ldcg(&cs->status);
      rr.n_records = __ldcg(&cs->nr);
      rr.n_frags = __ldcg(&cs->kept);
      rr.consumed = __ldcg(&cs->consumed);
    } else {
      rr.status = __ldcg(&pl->end.status);
      rr.n_records = __ldcg(&pl->end.n_records);
      rr.n_frags = __ldcg(&pl->end.n_frags);
      rr.consumed = __ldcg(&pl->end.consumed);
    }
    rr.rec_base = 0;
    rr.reply_bytes = 0;
    ix.res[r] = rr;
  }
  pl->ticket_b = 0;
  pl->stop_key = ~0ull;
  pl->fallback = 0;
}

// Ring r is final: the last ring of the launch numbers the records densely across rings.  One thread.
__device__ void ring_done(const IndexDev& ix, uint32_t n_rings) {
  __threadfence();
  if (atomicAdd(ix.ticket, 1u) == n_rings - 1) {
    __threadfence();
    dense_numbering(ix, n_rings);
    *ix.ticket = 0;
  }
}

__global__ void __launch_bounds__(kThreads) chunk_walk_kernel(IndexDev ix, ChunkParam P, ConfigDev cfg) {
  pdl_entry();
  TL_BEGIN(cfg, TL_SCAN);
  extern __shared__ __align__(128) uint8_t zone[];
  __shared__ SelSmem M;
  __shared__ ScanState S;
  __shared__ ResSmem RS;
  __shared__ uint64_t cand[kCand];
  __shared__ uint32_t ncand, last;
  uint32_t r, i, K;
  MTRACE(0);
  locate(P, blockIdx.x, r, i, K);
  const RingDesc R = P.r[r];
  if (K == 1) {  // a short window: the one-CTA scan
    scan_ring_cta(ix, R, false, r, cfg, S);
    if (threadIdx.x == 0) ring_done(ix, P.n_rings);
    TL_END(cfg, TL_SCAN);
    return;
  }
  const uint64_t ci = R.head + (uint64_t)i * P.S[r];
  const uint64_t cn = i + 1 == K ? R.tail : ci + P.S[r];
  if (i == 0) {
    if (threadIdx.x == 0) {
      ix.rings[r] = R;
      cand[0] = R.head;
      ncand = 1;
    }
  } else {
    const uint32_t nc = select_candidates(R, ci, cn, zone, M, cand);
    if (threadIdx.x == 0) ncand = nc;
  }
  __syncthreads();
  MTRACE(4);
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = blockIdx.x;
  if (warp < kCand) {
    ChainSum* cs = ix.ms.sums + (uint64_t)g * kCand + warp;
    if (warp < ncand) {
      walk_chain(R, cand[warp], ci, cn, cfg.guess, ix.ms.log + ((uint64_t)g * kCand + warp) * kLogCap, cs, lane);
    } else if (lane == 0) {
      ChainSum z{};
      z.start = ~0ull;
      z.pad_ = 0;
      z.kind = CH_NONE;
      *cs = z;
    }
  }
  __syncthreads();
  MTRACE(5);
  if (threadIdx.x == 0) {
    __threadfence();
    last = atomicAdd(&ix.ms.plan[r].ticket_a, 1u) == K - 1;
  }
  __syncthreads();
  if (last) {
    __threadfence();
    resolve_ring(ix, P, r, K, R, RS, zone);
    if (K <= kInlineChunks) {  // a ring of few chunks is emitted here: its warps take the chunks in turn
      __syncthreads();
      const bool fb = __ldcg(&ix.ms.plan[r].fallback) != 0;
      if (fb) {
        scan_ring_cta(ix, R, false, r, cfg, S);  // no candidate fitted: the one-CTA scan of the whole window
      } else {
        for (uint32_t c = warp; c < K; c += blockDim.x >> 5) emit_chunk(ix, P, cfg, r, c, P.chunk0[r] + c, R, lane);
        __syncthreads();
      }
      if (threadIdx.x == 0) {
        __threadfence();
        finalize_ring(ix, r, fb);
        ring_done(ix, P.n_rings);
      }
    }
  }
  MTRACE(6);
  TL_END(cfg, TL_SCAN);
}

// Emission of chunk g's true chain (warp 0) from its entry state.
__device__ void emit_chunk(const IndexDev& ix, const ChunkParam& P, const ConfigDev& cfg, uint32_t r, uint32_t i,
                           uint32_t g, const RingDesc& R, uint32_t lane) {
  const ChunkState* sp = ix.ms.state + g;
  const int32_t chosen = __ldcg(&sp->chosen);
  if (chosen < 0) return;
  const ChainSum cs = ld_sum(ix.ms.sums + (uint64_t)g * kCand + chosen);
  const uint2* log = ix.ms.log + ((uint64_t)g * kCand + chosen) * kLogCap;
  const uint64_t ci = R.head + (uint64_t)i * P.S[r];
  const uint32_t FC = ix.frags_per_ring, RC = ix.recs_per_ring;
  const Env E{ix, R, cfg.max_record_bytes, (uint64_t)r * FC, (uint64_t)r * RC, FC, RC};
  Walk W{__ldcg(&sp->p), __ldcg(&sp->r0), __ldcg(&sp->sum), __ldcg(&sp->nf), __ldcg(&sp->nr), __ldcg(&sp->f0),
         0, 0, false, 0, 0, 0};
  for (uint32_t k0 = __ldcg(&sp->skip); k0 < cs.n; k0 += 32) {
    const uint32_t nt = min(32u, cs.n - k0);
    const uint2 e = lane < nt ? __ldcg(log + k0 + lane) : make_uint2(0, 0);
    const uint32_t nf0 = W.nf;
    const int tf = take_hops(E, W, lane, nt, ci + e.x, e.y);
    if (tf >= 0) {  // a check failed at hop tf: its outcome, keyed by its fragment number
      if (lane == 0) {
        ChunkStop st;
        st.consumed = W.consumed;
        st.status = W.status;
        st.nr = W.nr;
        st.kept = W.kept;
        st.pad_ = 0;
        ix.ms.stops[g] = st;
        __threadfence();
        atomicMin(&ix.ms.plan[r].stop_key, ((unsigned long long)(nf0 + (uint32_t)tf) << 24) | g);
      }
      return;
    }
  }
}

// Rings of more than kInlineChunks chunks: one CTA per chunk emits it; the ring's last CTA finalizes it.
__global__ void __launch_bounds__(kThreads) chunk_emit_kernel(IndexDev ix, ChunkParam P, ConfigDev cfg) {
  pdl_entry();
  TL_BEGIN(cfg, TL_SCAN);
  __shared__ ScanState S;
  __shared__ uint32_t last, fb;
  uint32_t r, i, K;
  locate(P, blockIdx.x, r, i, K);
  if (K <= kInlineChunks) {  // one-CTA rings and rings emitted by their resolver are final already
    TL_END(cfg, TL_SCAN);
    return;
  }
  const RingDesc R = P.r[r];
  RingPlan* pl = ix.ms.plan + r;
  if (threadIdx.x == 0) fb = __ldcg(&pl->fallback);
  __syncthreads();
  if (fb) {
    if (i == 0) scan_ring_cta(ix, R, false, r, cfg, S);  // the one-CTA scan of the whole window
  } else if (threadIdx.x < 32) {
    emit_chunk(ix, P, cfg, r, i, blockIdx.x, R, threadIdx.x);
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    last = atomicAdd(&pl->ticket_b, 1u) == K - 1;
    if (last) {
      __threadfence();
      finalize_ring(ix, r, fb != 0);
      ring_done(ix, P.n_rings);
    }
  }
  TL_END(cfg, TL_SCAN);
}

cudaError_t ensure_walk_smem() {
  static std::mutex mu;
  static bool set[kMaxDevices] = {};
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= kMaxDevices) return cudaErrorInvalidDevice;
  std::lock_guard<std::mutex> lk(mu);
  if (set[dev]) return cudaSuccess;
  e = cudaFuncSetAttribute(chunk_walk_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kZoneBytes);
  if (e == cudaSuccess) set[dev] = true;
  return e;
}

}  // namespace

#ifdef CRK_MSCAN_TRACE
extern "C" int crk_debug_mscan_trace(unsigned long long* out) {
  return cudaMemcpyFromSymbol(out, g_mtrace, sizeof(g_mtrace)) == cudaSuccess ? 0 : -100;
}
#endif

// Chunk plan: the chunk size S (a power of two, >= 256 KiB) gives the launch about 2 chunks per SM over the
// total window; a ring gets floor(window / S) chunks of ceil(window / chunks) bytes (16-byte multiples), one
// when its window is shorter than 2 S.  False when no ring has two chunks (the one-CTA scan serves them all).
bool chunk_plan(const IndexDev& ix, const ScanRingsParam& p, int sms, void* out_param) {
  ChunkParam& P = *static_cast<ChunkParam*>(out_param);
  if (p.doorbell || p.n_rings == 0) return false;
  uint64_t total = 0;
  for (uint32_t r = 0; r < p.n_rings; ++r) total += p.r[r].tail - p.r[r].head;
  const uint64_t target = 2ull * (uint64_t)(sms > 0 ? sms : 148);  // one wave: 2 K1a CTAs fit an SM
  uint64_t S = 256 * 1024;
  while (S * target < total) S <<= 1;
  for (;;) {
    uint32_t acc = 0;
    bool multi = false, fits = true;
    for (uint32_t r = 0; r < p.n_rings; ++r) {
      const uint64_t W = p.r[r].tail - p.r[r].head;
      uint64_t K = W >= 2 * S ? W / S : 1;
      if (K > kMaxRingChunks) { fits = false; break; }
      P.chunk0[r] = acc;
      P.S[r] = K > 1 ? ((W + K - 1) / K + 15) & ~15ull : W;
      acc += (uint32_t)K;
      multi |= K > 1;
    }
    if (fits && acc <= ix.ms.chunk_cap) {
      if (!multi || S > (1ull << 31)) return false;  // logs keep cursors as 32-bit offsets into the chunk
      P.chunk0[p.n_rings] = acc;
      P.n_rings = p.n_rings;
      P.need_emit = 0;
      for (uint32_t r = 0; r < p.n_rings; ++r) P.need_emit |= P.chunk0[r + 1] - P.chunk0[r] > kInlineChunks;
      for (uint32_t r = 0; r < p.n_rings; ++r) P.r[r] = p.r[r];
      return true;
    }
    S <<= 1;
  }
}

uint32_t chunk_plan_chunks(const void* param) {
  const ChunkParam& P = *static_cast<const ChunkParam*>(param);
  return P.chunk0[P.n_rings];
}

size_t chunk_param_bytes() { return sizeof(ChunkParam); }

cudaError_t launch_chunk_scan(const IndexDev& ix, const void* param, const ConfigDev& cfg, cudaStream_t s) {
  const ChunkParam& P = *static_cast<const ChunkParam*>(param);
  cudaError_t e = ensure_walk_smem();
  if (e != cudaSuccess) return e;
  const uint32_t n = P.chunk0[P.n_rings];
  CRK_LAUNCH(pdl_of(cfg), chunk_walk_kernel, n, kThreads, kZoneBytes, s, ix, P, cfg);
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  if (P.need_emit) CRK_LAUNCH(pdl_of(cfg), chunk_emit_kernel, n, kThreads, 0, s, ix, P, cfg);
  return cudaGetLastError();
}

}  // namespace crk
