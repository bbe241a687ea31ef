// Logical-record access: byte o of a record is byte (o - lstart[k]) of the fragment k that holds it
// (RFC 5531 §11: the record is the concatenation of its fragments).  Used by the parser and by the
// movers' per-byte edge paths; the bulk paths never call it per byte.
#pragma once
#include "crk_device.cuh"

namespace crk {

struct LogicalRecord {
  RingDesc R;
  const uint64_t* phys;
  const uint64_t* lstart;
  const uint32_t* hdr;
  uint32_t nfrags;
  uint32_t frag0;  // absolute index of the first fragment
  uint32_t hint;
  uint64_t len;
  uint64_t F0;

  __device__ __forceinline__ void init(const IndexDev& ix, const RingDesc& r, uint32_t slot) {
    R = r;
    const uint32_t f0 = ix.rec_frag0[slot];
    frag0 = f0;
    nfrags = ix.rec_nfrags[slot];
    len = ix.rec_len[slot];
    phys = ix.frag_phys + f0;
    lstart = ix.frag_lstart + f0;
    hdr = ix.frag_hdr + f0;
    hint = 0;
    F0 = hdr[0] & 0x7fffffffu;
  }
  __device__ __forceinline__ uint64_t flen(uint32_t k) const { return hdr[k] & 0x7fffffffu; }
  __device__ __forceinline__ bool holds(uint32_t k, uint64_t off) const {
    const uint64_t ls = lstart[k];
    return off >= ls && off < ls + flen(k);
  }
  // Fragment holding logical byte `off` (< len): the hint, its next fragments, the uniform-stride
  // guess off / F0, then binary search for the largest k with lstart[k] <= off.
  __device__ uint32_t find(uint64_t off) {
    uint32_t k = hint;
    if (k < nfrags && holds(k, off)) return k;
    for (uint32_t i = 1; i <= 3 && k + i < nfrags; ++i)
      if (holds(k + i, off)) return hint = k + i;
    if (F0 > 0) {
      uint64_t g = off / F0;
      if (g < nfrags && holds((uint32_t)g, off)) return hint = (uint32_t)g;
    }
    uint32_t lo = 0, hi = nfrags;  // invariant: lstart[lo] <= off, and lstart[hi] > off or hi == nfrags
    while (hi - lo > 1) {
      uint32_t mid = (lo + hi) >> 1;
      if (lstart[mid] <= off) lo = mid; else hi = mid;
    }
    return hint = lo;
  }
  __device__ __forceinline__ uint8_t byte(uint64_t off) {
    const uint32_t k = find(off);
    return ring_byte(R, phys[k] + (off - lstart[k]));
  }
  __device__ __forceinline__ uint32_t be32(uint64_t off) {
    const uint32_t k = find(off);
    const uint64_t rel = off - lstart[k];
    if (rel + 4 <= flen(k)) return ring_be32(R, phys[k] + rel);
    return ((uint32_t)byte(off) << 24) | ((uint32_t)byte(off + 1) << 16) | ((uint32_t)byte(off + 2) << 8) |
           (uint32_t)byte(off + 3);
  }
};

}  // namespace crk
