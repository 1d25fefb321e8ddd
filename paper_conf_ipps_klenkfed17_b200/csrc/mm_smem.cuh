// mm_smem.cuh -- shared-memory building blocks of the per-endpoint / per-bucket
// matching kernels: 16-bit atomics through 32-bit words, ballot-based peer
// masks and warp-ordered placement into per-tuple lists.
#pragma once

#include "mm_internal.cuh"

namespace mm {

constexpr uint16_t kWild = 0xFFFEu;
constexpr uint16_t kNone = 0xFFFFu;
constexpr uint16_t kEmpty16 = 0xFFFFu;
constexpr uint16_t kPending16 = 0xFFFEu;  // slot claimed, id not yet published

// Slot of a tuple in an on-chip hash table: multiply-shift of the 64-bit word
// (a few instructions; the tables are small and private to one CTA).
__device__ __forceinline__ uint32_t slot_hash(uint64_t h) {
  return (uint32_t)((h * 0xD6E8FEB86659FD93ull) >> 40);
}

// 16-bit CAS through the containing 32-bit word.
// (pointer arithmetic, not integer casts, so shared-memory provenance survives
// and the atomics compile to ATOMS)
__device__ __forceinline__ uint32_t* word_of(uint16_t* p) {
  return reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(p) - (reinterpret_cast<uintptr_t>(p) & 2));
}
__device__ __forceinline__ uint16_t cas16(uint16_t* p, uint16_t expect, uint16_t val) {
  uint32_t* w = word_of(p);
  const uint32_t sh = (reinterpret_cast<uintptr_t>(p) & 2) ? 16u : 0u;
  uint32_t old = *w;
  while (true) {
    const uint16_t cur = (uint16_t)(old >> sh);
    if (cur != expect) return cur;
    const uint32_t nw = (old & ~(0xFFFFu << sh)) | ((uint32_t)val << sh);
    const uint32_t got = atomicCAS(w, old, nw);
    if (got == old) return expect;
    old = got;
  }
}

// 16-bit exchange through the containing 32-bit word.
__device__ __forceinline__ uint16_t exch16(uint16_t* p, uint16_t v) {
  uint32_t* w = word_of(p);
  const uint32_t sh = (reinterpret_cast<uintptr_t>(p) & 2) ? 16u : 0u;
  uint32_t old = *w;
  while (true) {
    const uint32_t nw = (old & ~(0xFFFFu << sh)) | ((uint32_t)v << sh);
    const uint32_t got = atomicCAS(w, old, nw);
    if (got == old) return (uint16_t)(old >> sh);
    old = got;
  }
}

// 16-bit counter increment through the containing 32-bit word (no carry out:
// counts stay below 65536).
__device__ __forceinline__ void inc16(uint16_t* p) {
  atomicAdd(word_of(p), (reinterpret_cast<uintptr_t>(p) & 2) ? 0x10000u : 1u);
}
// Same, returning the previous 16-bit value.
__device__ __forceinline__ uint32_t fetch_inc16(uint16_t* p) {
  const bool hi = (reinterpret_cast<uintptr_t>(p) & 2) != 0;
  const uint32_t old = atomicAdd(word_of(p), hi ? 0x10000u : 1u);
  return hi ? (old >> 16) : (old & 0xFFFFu);
}

// Lanes holding the same value as this lane: one match.any.sync (measured on
// B200 at a constant ~200 cycles of latency whatever the number of distinct
// values, 2-3x cheaper than one ballot per value bit; tools/micro/peers.cu).
__device__ __forceinline__ uint32_t peers_of(uint32_t v) { return __match_any_sync(kFull, v); }

#ifndef MM_P6_PIPE
#define MM_P6_PIPE 0  // A/B: 17.55 vs 17.62 G matches/s on configs[1] (rejected)
#endif
// Ordered placement by one warp: element x (0..n) with tuple id key(x) (>=
// kWild = skip) gets slot start[k] + running[k]; put(x, k, rank, slot).
// nkeys bounds the tuple ids (ids < nkeys).
template <class KeyF, class PutF>
__device__ __forceinline__ void place_in_order(int64_t n, KeyF key, const uint16_t* start, uint16_t* running, PutF put,
                                               int lane, uint32_t lt, uint32_t nkeys) {
#if MM_P6_PIPE
  // software-pipelined: the next chunk's keys and peer masks (match.any,
  // ~200 cycles) are requested before this chunk's running counts are read
  // and advanced, so the peer latency overlaps the dependent count chain
  uint32_t kn = lane < n ? key(lane) : 0xFFFFFFFFu;
  uint32_t pn = peers_of(kn < kWild ? kn : nkeys);
  for (int64_t b = 0; b < n; b += 32) {
    const int64_t x = b + lane;
    const uint32_t k = kn, peers = pn;
    const bool ok = k < kWild;
    if (b + 32 < n) {
      kn = x + 32 < n ? key(x + 32) : 0xFFFFFFFFu;
      pn = peers_of(kn < kWild ? kn : nkeys);
    }
    uint32_t run = 0;
#else
  for (int64_t b = 0; b < n; b += 32) {
    const int64_t x = b + lane;
    const uint32_t k = x < n ? key(x) : 0xFFFFFFFFu;
    const bool ok = k < kWild;
    const uint32_t peers = peers_of(ok ? k : nkeys);  // nkeys = "skip"
    uint32_t run = 0;
#endif
    if (ok) run = running[k];
    __syncwarp();
    if (ok) {
      const uint32_t r = run + __popc(peers & lt);
      put(x, k, r, (uint32_t)start[k] + r);
      if ((peers >> lane) == 1u) running[k] = (uint16_t)(run + __popc(peers));
    }
    __syncwarp();
  }
}

}  // namespace mm
