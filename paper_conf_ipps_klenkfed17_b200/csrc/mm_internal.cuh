// mm_internal.cuh -- device utilities shared by the matching kernels.
//
// Product code (sm_100a).  Shares nothing with oracle/ (DESIGN.md §4).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/mm.h"

namespace mm {

constexpr uint32_t kFull = 0xFFFFFFFFu;
constexpr int kScanThreads = 256;
constexpr int kScanItems = 16;
constexpr int kScanTile = kScanThreads * kScanItems;  // 4096 elements per CTA tile

// Process-wide count of kernel launches issued by this library (host side,
// reported through mm_query's MM_Q_LAUNCHES).
long long& launch_count();
inline void count_launch(int n = 1) { launch_count() += n; }

// Sticky device error bits (mm_query reports MM_ERR_CAPACITY if any is set).
enum : uint32_t { kErrCapacity = 1u, kErrOutput = 2u };

// ------------------------------------------------------------------ header
// Header word (include/mm.h): src 0..31, tag 32..47, comm 48..63.
// Admissibility under full MPI semantics (§II.B l.65) is one masked
// XOR: the receive's wildcard fields are cleared from the comparison mask.
__device__ __forceinline__ uint64_t wildcard_mask(uint64_t r) {
  uint64_t m = ~0ull;
  if ((uint32_t)r == MM_ANY_SOURCE) m &= ~0xFFFFFFFFull;
  if (((uint32_t)(r >> 32) & 0xFFFFu) == MM_ANY_TAG) m &= ~(0xFFFFull << 32);
  return m;
}

// Robert Jenkins' 32-bit integer hash, 6-shift variant (§VI.C l.219).
__device__ __forceinline__ uint32_t jenkins32(uint32_t a) {
  a = (a + 0x7ed55d16u) + (a << 12);
  a = (a ^ 0xc761c23cu) ^ (a >> 19);
  a = (a + 0x165667b1u) + (a << 5);
  a = (a + 0xd3a2646cu) ^ (a << 9);
  a = (a + 0xfd7046c5u) + (a << 3);
  a = (a ^ 0xb55a4f09u) ^ (a >> 16);
  return a;
}
// 64-bit header folded into the 32-bit hash (reading R7).
__device__ __forceinline__ uint32_t header_hash(uint64_t h) {
  return jenkins32((uint32_t)h ^ jenkins32((uint32_t)(h >> 32)));
}

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// --------------------------------------------------------------- snapshot
// A batch snapshot of one queue side: residual queue entries first, then the
// pending (posted but not yet matched) elements (§V l.128).
struct Side {
  const uint64_t* q_hdr;    // residual headers (queue storage)
  const int64_t* q_cookie;  // residual cookies
  const int32_t* q_len;     // residual length per endpoint (device)
  const uint64_t* p_hdr;    // pending headers (nullptr if none)
  const int64_t* p_cookie;  // pending cookies (nullptr -> p_seq0 + index)
  const int64_t* p_off;     // pending CSR offsets (nullptr -> single endpoint)
  int64_t p_n;              // pending element count
  int64_t p_seq0;           // cookie of the first pending element if p_cookie == nullptr
  int64_t cap;              // queue capacity per endpoint (stride)

  __device__ __forceinline__ int64_t pend_begin(int e) const { return p_hdr ? (p_off ? p_off[e] : 0) : 0; }
  __device__ __forceinline__ int64_t pend_count(int e) const {
    if (!p_hdr) return 0;
    return p_off ? p_off[e + 1] - p_off[e] : p_n;
  }
  // k-th snapshot element of endpoint e (resid = q_len[e], pb = pend_begin(e))
  __device__ __forceinline__ uint64_t hdr(int e, int64_t k, int64_t resid, int64_t pb) const {
    return k < resid ? q_hdr[(int64_t)e * cap + k] : p_hdr[pb + (k - resid)];
  }
  __device__ __forceinline__ int64_t cookie(int e, int64_t k, int64_t resid, int64_t pb) const {
    if (k < resid) return q_cookie[(int64_t)e * cap + k];
    int64_t i = pb + (k - resid);
    return p_cookie ? p_cookie[i] : p_seq0 + i;
  }
};

// One endpoint's snapshot side with the per-endpoint address arithmetic done
// once: element k < resid is queue entry k, element k >= resid pending entry
// k - resid (the pending pointers are pre-offset by -resid).
#ifndef MM_EPSIDE_SEL
#define MM_EPSIDE_SEL 1  // A/B: configs[1] 17.74 vs 17.61 G matches/s (fewer instructions per header access)
#endif
struct EpSide {
  const uint64_t* qh;
  const int64_t* qc;
  const uint64_t* ph;
  const int64_t* pc;
  int64_t cseq;  // computed cookie of pending element k: cseq + k
  uint32_t resid;
  __device__ __forceinline__ EpSide(const Side& S, int e, int64_t res, int64_t pb) {
    qh = S.q_hdr + (int64_t)e * S.cap;
    qc = S.q_cookie + (int64_t)e * S.cap;
    ph = S.p_hdr ? S.p_hdr + (pb - res) : nullptr;
    pc = S.p_cookie ? S.p_cookie + (pb - res) : nullptr;
    cseq = S.p_seq0 + pb - res;
    resid = (uint32_t)res;
  }
#if MM_EPSIDE_SEL
  // (the base pointer selected, then one load)
  __device__ __forceinline__ uint64_t hdr(uint32_t k) const { return (k < resid ? qh : ph)[k]; }
#else
  __device__ __forceinline__ uint64_t hdr(uint32_t k) const { return k < resid ? qh[k] : ph[k]; }
#endif
  __device__ __forceinline__ int64_t cookie(uint32_t k) const {
    if (k < resid) return qc[k];
    return pc ? pc[k] : cseq + (int64_t)k;
  }
};

// ------------------------------------------------------------ block scans
template <class T>
__device__ __forceinline__ T warp_incl_scan(T v) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T t = __shfl_up_sync(kFull, v, o);
    if (lane >= o) v += t;
  }
  return v;
}

// Exclusive block scan of one value per thread; returns the block total in
// *total.  `sm` must hold blockDim.x/32 + 1 elements.
template <class T>
__device__ __forceinline__ T block_excl_scan(T v, T* sm, T* total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  T inc = warp_incl_scan(v);
  if (lane == 31) sm[w] = inc;
  __syncthreads();
  if (w == 0) {
    T x = lane < nw ? sm[lane] : T(0);
    T xi = warp_incl_scan(x);
    if (lane < nw) sm[lane] = xi - x;
    if (lane == nw - 1) sm[nw] = xi;
  }
  __syncthreads();
  T r = sm[w] + inc - v;
  *total = sm[nw];
  __syncthreads();
  return r;
}

// ------------------------------------------------- device-wide exclusive scan
// Three phases: per-tile reduce, scan of tile sums (one CTA), per-tile
// downsweep that hands (index, exclusive prefix, value) to a functor, so the
// consumer (compaction, run boundaries) is fused into the last pass.
template <class T, class In>
__global__ void __launch_bounds__(kScanThreads) k_tile_reduce(In in, int64_t n, T* tile_sums) {
  __shared__ T sm[kScanThreads / 32 + 1];
  int64_t base = (int64_t)blockIdx.x * kScanTile + threadIdx.x;
  T s = 0;
#pragma unroll
  for (int i = 0; i < kScanItems; i++) {
    int64_t k = base + (int64_t)i * kScanThreads;
    if (k < n) s += in(k);
  }
  T tot;
  block_excl_scan(s, sm, &tot);
  if (threadIdx.x == 0) tile_sums[blockIdx.x] = tot;
}

// In-place exclusive scan of a[0..n) by one CTA; a[n] receives the total.
template <class T>
__global__ void __launch_bounds__(1024) k_scan_single(T* a, int64_t n) {
  __shared__ T sm[1024 / 32 + 1];
  T carry = 0;
  for (int64_t b = 0; b < n; b += 1024) {
    int64_t k = b + threadIdx.x;
    T v = k < n ? a[k] : T(0);
    T tot;
    T ex = block_excl_scan(v, sm, &tot);
    if (k < n) a[k] = carry + ex;
    carry += tot;
  }
  if (threadIdx.x == 0) a[n] = carry;
}

// Downsweep: element k (< n) with exclusive prefix p calls out(k, p, v).
// Items are processed in "blocked" order per thread so that the prefix of a
// thread's items is sequential.
template <class T, class In, class Out>
__global__ void __launch_bounds__(kScanThreads) k_tile_downsweep(In in, int64_t n, const T* tile_off, Out out) {
  __shared__ T sm[kScanThreads / 32 + 1];
  const int64_t tbase = (int64_t)blockIdx.x * kScanTile;
  T v[kScanItems];
  T s = 0;
#pragma unroll
  for (int i = 0; i < kScanItems; i++) {
    int64_t k = tbase + (int64_t)threadIdx.x * kScanItems + i;
    v[i] = k < n ? in(k) : T(0);
    s += v[i];
  }
  T tot;
  T p = block_excl_scan(s, sm, &tot) + tile_off[blockIdx.x];
#pragma unroll
  for (int i = 0; i < kScanItems; i++) {
    int64_t k = tbase + (int64_t)threadIdx.x * kScanItems + i;
    if (k < n) out(k, p, v[i]);
    p += v[i];
  }
}

// k_tile_reduce sums tiles of 4096 contiguous elements in strided order and
// k_tile_downsweep visits the same tile in blocked order: both cover exactly
// [tile*4096, tile*4096+4096), so the tile offsets agree.
template <class T, class In, class Out>
cudaError_t scan_apply(In in, int64_t n, T* scratch /* >= ntiles + 1 */, Out out, cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  int64_t nt = (n + kScanTile - 1) / kScanTile;
  count_launch(3);
  k_tile_reduce<T, In><<<(unsigned)nt, kScanThreads, 0, st>>>(in, n, scratch);
  k_scan_single<T><<<1, 1024, 0, st>>>(scratch, nt);
  k_tile_downsweep<T, In, Out><<<(unsigned)nt, kScanThreads, 0, st>>>(in, n, scratch, out);
  return cudaGetLastError();
}

inline int64_t scan_scratch_elems(int64_t n) { return (n + kScanTile - 1) / kScanTile + 2; }

// Host-side launch helpers: the dynamic shared-memory opt-in and the
// occupancy of a kernel are fixed per (kernel, device), so they are queried
// once instead of on every launch (each call costs microseconds of host time
// on the batch's critical path).
template <auto KERNEL>
inline cudaError_t ensure_dyn_smem(size_t bytes) {
  static int allowed[64] = {0};
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) {
    cudaGetLastError();
    return cudaFuncSetAttribute(KERNEL, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
  }
  if ((int)bytes <= allowed[dev]) return cudaSuccess;
  const cudaError_t err = cudaFuncSetAttribute(KERNEL, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
  if (err == cudaSuccess) allowed[dev] = (int)bytes;
  return err;
}

// resident CTAs of KERNEL on the whole chip (SMs x blocks per SM), cached per
// (kernel, device): every launch of a kernel uses one block size and one
// dynamic shared-memory size
template <auto KERNEL>
inline int resident_ctas(int threads, size_t smem) {
  static int cached[64] = {0};
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) {
    cudaGetLastError();
    dev = -1;
  }
  if (dev >= 0 && cached[dev] > 0) return cached[dev];
  int sms = 148, occ = 1;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev < 0 ? 0 : dev) != cudaSuccess ||
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, KERNEL, threads, smem) != cudaSuccess) {
    cudaGetLastError();
    sms = 148;
    occ = 1;
  }
  const int r = sms * (occ < 1 ? 1 : occ);
  if (dev >= 0) cached[dev] = r;
  return r;
}

// ---------------------------------------------- stable bucket partition
// Stable counting-sort scatter of n elements into up to 512 buckets.  Used by
// the LSD radix passes of the ordered no-wildcard level (row A4) and by
// mm_route (row A6).  Tile = 8 warps x 512 contiguous elements; each warp owns
// a contiguous chunk and keeps private running counts per bucket, so ranks are
// stable without CTA-wide barriers inside the tile.
constexpr int kPartWarps = 8;
constexpr int kPartThreads = kPartWarps * 32;
constexpr int kPartItems = 6;                           // per lane
constexpr int kPartMaxBuckets = 512;
constexpr int kPartWarpChunk = 32 * kPartItems;         // 256 elements per warp
constexpr int kPartTile = kPartWarps * kPartWarpChunk;  // 2048 elements per tile

// hist[b * ntiles + tile] = elements of tile with bucket b.
template <class BucketF>
__global__ void __launch_bounds__(kPartThreads) k_part_hist(BucketF bucket, int64_t n, int nbuckets, int64_t ntiles,
                                                            uint32_t* hist) {
  __shared__ uint32_t h[kPartMaxBuckets];
  for (int b = threadIdx.x; b < kPartMaxBuckets; b += blockDim.x) h[b] = 0;
  __syncthreads();
  const int64_t base = (int64_t)blockIdx.x * kPartTile;
  constexpr int kPer = kPartTile / kPartThreads;  // elements per thread, all loads in flight
  uint32_t bk[kPer];
#pragma unroll
  for (int j = 0; j < kPer; j++) {
    const int64_t k = base + threadIdx.x + j * kPartThreads;
    bk[j] = k < n ? bucket(k) : 0xFFFFFFFFu;
  }
#pragma unroll
  for (int j = 0; j < kPer; j++)
    if (bk[j] != 0xFFFFFFFFu) atomicAdd(&h[bk[j]], 1u);
  __syncthreads();
  for (int b = threadIdx.x; b < nbuckets; b += blockDim.x) hist[(int64_t)b * ntiles + blockIdx.x] = h[b];
}

// Scatter: element k of bucket b goes to off[b * ntiles + tile] + its rank
// among the tile's bucket-b elements in input order.  The payload moves
// through shared memory: elements are first placed in tile-local bucket order,
// then written out so that consecutive threads write consecutive addresses of
// a bucket's run (coalesced stores instead of one scattered store per lane).
// move.load(k, a, b) reads element k's payload, move.store(dst, a, b) writes it.
#ifndef MM_PART_ALWAYS_SENTINEL
#define MM_PART_ALWAYS_SENTINEL 0  // 1: ten ballots per item everywhere (the previous scheme, for A/B)
#endif
#ifndef MM_PART_MIN_BLOCKS
#define MM_PART_MIN_BLOCKS 4  // resident scatter CTAs per SM the register budget must allow (3: -6 %)
#endif
constexpr size_t kPartSmem = (size_t)kPartTile * (8 + 8 + 2) + (kPartWarps + 2) * kPartMaxBuckets * 4 + 64 * 4 + 16;

// BITS: digit width (nbuckets <= 2^BITS): a full tile needs exactly BITS
// ballots per item; the tail tile adds the sentinel bit for invalid lanes.
template <class BucketF, class MoveF, int BITS>
__global__ void __launch_bounds__(kPartThreads, MM_PART_MIN_BLOCKS) k_part_scatter(BucketF bucket, MoveF move, int64_t n, int nbuckets,
                                                               int64_t ntiles, const uint32_t* off) {
  extern __shared__ __align__(16) uint8_t part_smem[];
  uint64_t* sa = reinterpret_cast<uint64_t*>(part_smem);
  uint64_t* sb = sa + kPartTile;
  uint32_t* wrun = reinterpret_cast<uint32_t*>(sb + kPartTile);  // [kPartWarps][kPartMaxBuckets]
  uint32_t* lstart = wrun + kPartWarps * kPartMaxBuckets;         // tile-local bucket starts
  uint32_t* gbase = lstart + kPartMaxBuckets;                     // global bucket bases
  uint32_t* scan_sm = gbase + kPartMaxBuckets;
  uint16_t* sbk = reinterpret_cast<uint16_t*>(scan_sm + 64);
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int b = lane; b < kPartMaxBuckets; b += 32) wrun[w * kPartMaxBuckets + b] = 0;
  for (int b = threadIdx.x; b < nbuckets; b += blockDim.x) gbase[b] = off[(int64_t)b * ntiles + blockIdx.x];
  __syncwarp();
  const int64_t tbase = (int64_t)blockIdx.x * kPartTile;
  const int64_t cbase = tbase + (int64_t)w * kPartWarpChunk;
  const bool full = tbase + kPartTile <= n;  // CTA-uniform
  const uint32_t lt = lanemask_lt();
  uint32_t rank[kPartItems];
  uint32_t bk[kPartItems];
  uint64_t va[kPartItems], vb[kPartItems];
  // all loads of the chunk in flight before the first use (the ballots and
  // __syncwarp below would otherwise serialise one HBM round trip per item)
#pragma unroll
  for (int r = 0; r < kPartItems; r++) {
    const int64_t k = cbase + r * 32 + lane;
    va[r] = 0;
    vb[r] = 0;
    if (k < n) move.load(k, va[r], vb[r]);
  }
#pragma unroll
  for (int r = 0; r < kPartItems; r++) {
    int64_t k = cbase + r * 32 + lane;
    bool valid = k < n;
    uint32_t b = 0;
    if (valid) b = bucket.of_payload(k, va[r], vb[r]);
    // lanes with the same bucket: one ballot per digit bit (with several
    // items in flight, cheaper than match.any); in the tail tile invalid
    // lanes carry the sentinel value 2^BITS (one more ballot)
    uint32_t peers = kFull;
    if (full && !MM_PART_ALWAYS_SENTINEL) {
#pragma unroll
      for (int bit = 0; bit < BITS; bit++) {
        const bool x = (b >> bit) & 1u;
        const uint32_t bb = __ballot_sync(kFull, x);
        peers &= x ? bb : ~bb;
      }
    } else {
      const uint32_t v = valid ? b : (1u << BITS);
#pragma unroll
      for (int bit = 0; bit <= BITS; bit++) {
        const bool x = (v >> bit) & 1u;
        const uint32_t bb = __ballot_sync(kFull, x);
        peers &= x ? bb : ~bb;
      }
    }
    uint32_t before = wrun[w * kPartMaxBuckets + b];
    __syncwarp();
    if (valid) {
      rank[r] = before + __popc(peers & lt);
      // the highest peer lane publishes the new running count
      if ((peers >> lane) == 1u) wrun[w * kPartMaxBuckets + b] = before + __popc(peers);
    }
    bk[r] = valid ? b : 0xFFFFFFFFu;
    __syncwarp();
  }
  __syncthreads();
  // tile-local bucket starts and per-warp offsets (thread t: buckets 2t, 2t+1)
  {
    constexpr int BPT = kPartMaxBuckets / kPartThreads;
    uint32_t tot[BPT];
    uint32_t sum = 0;
#pragma unroll
    for (int j = 0; j < BPT; j++) {
      const int b = threadIdx.x * BPT + j;
      tot[j] = 0;
      if (b < nbuckets)
        for (int ww = 0; ww < kPartWarps; ww++) tot[j] += wrun[ww * kPartMaxBuckets + b];
      sum += tot[j];
    }
    uint32_t all;
    uint32_t ls = block_excl_scan<uint32_t>(sum, scan_sm, &all);
#pragma unroll
    for (int j = 0; j < BPT; j++) {
      const int b = threadIdx.x * BPT + j;
      if (b < nbuckets) {
        lstart[b] = ls;
        uint32_t sacc = ls;
        for (int ww = 0; ww < kPartWarps; ww++) {
          const uint32_t c = wrun[ww * kPartMaxBuckets + b];
          wrun[ww * kPartMaxBuckets + b] = sacc;
          sacc += c;
        }
      }
      ls += tot[j];
    }
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < kPartItems; r++) {
    if (bk[r] != 0xFFFFFFFFu) {
      const uint32_t lp = wrun[w * kPartMaxBuckets + bk[r]] + rank[r];
      sa[lp] = va[r];
      sb[lp] = vb[r];
      sbk[lp] = (uint16_t)bk[r];
    }
  }
  __syncthreads();
  const int64_t tn = n - tbase < kPartTile ? n - tbase : kPartTile;
  for (int t = threadIdx.x; t < tn; t += kPartThreads) {
    const uint32_t b = sbk[t];
    move.store((int64_t)gbase[b] + (t - lstart[b]), sa[t], sb[t]);
  }
}

struct ReadU32 {
  const uint32_t* a;
  __device__ __forceinline__ uint32_t operator()(int64_t k) const { return a[k]; }
};
struct WriteU32 {
  uint32_t* a;
  __device__ __forceinline__ void operator()(int64_t k, uint32_t p, uint32_t) const { a[k] = p; }
};

template <class BucketF, class MoveF>
cudaError_t partition_stable(BucketF bucket, MoveF move, int64_t n, int nbuckets, uint32_t* hist /* see partition_scratch_elems */,
                             cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  int64_t nt = (n + kPartTile - 1) / kPartTile;
  count_launch(2);
  k_part_hist<BucketF><<<(unsigned)nt, kPartThreads, 0, st>>>(bucket, n, nbuckets, nt, hist);
  // the bucket-major histogram is scanned in place (32-bit: n < 2^32)
  int64_t m = (int64_t)nbuckets * nt;
  // scan_apply needs separate scratch for tile sums: place it after the hist
  uint32_t* sc = hist + m + 1;
  cudaError_t err = scan_apply<uint32_t>(ReadU32{hist}, m, sc, WriteU32{hist}, st);
  if (err != cudaSuccess) return err;
  if (nbuckets <= 256 && !MM_PART_ALWAYS_SENTINEL) {
    err = ensure_dyn_smem<k_part_scatter<BucketF, MoveF, 8>>(kPartSmem);
    if (err != cudaSuccess) return err;
    k_part_scatter<BucketF, MoveF, 8><<<(unsigned)nt, kPartThreads, kPartSmem, st>>>(bucket, move, n, nbuckets, nt, hist);
    return cudaGetLastError();
  }
  err = ensure_dyn_smem<k_part_scatter<BucketF, MoveF, 9>>(kPartSmem);
  if (err != cudaSuccess) return err;
  k_part_scatter<BucketF, MoveF, 9><<<(unsigned)nt, kPartThreads, kPartSmem, st>>>(bucket, move, n, nbuckets, nt, hist);
  return cudaGetLastError();
}

inline int64_t partition_scratch_elems(int64_t n) {
  int64_t nt = (n + kPartTile - 1) / kPartTile;
  int64_t m = kPartMaxBuckets * nt;
  return m + 1 + scan_scratch_elems(m);
}

}  // namespace mm
