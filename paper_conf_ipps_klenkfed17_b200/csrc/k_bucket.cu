// k_bucket.cu -- the no-wildcard levels as hash-bucketed rank pairing
// (rows A4, A5 of DESIGN.md §1; §7.3).
//
// Without wildcards a receive can only take a message with the identical
// tuple, so the tuple key space partitions (§VI.A l.196; §VI.C
// l.215).  Both levels therefore
//  1. partition receives and messages by a hash of the tuple into B buckets of
//     ~1K elements with a STABLE counting-sort scatter (LSD over the bucket
//     bits, 8 bits per pass) -- stability keeps posting / arrival order inside
//     every bucket;
//  2. match every bucket in one CTA, entirely in shared memory: message tuples
//     get dense ids from a lock-free open-addressing table (32-bit CAS),
//     receives look their tuple up, and
//       - NOWILD_ORDERED (k_bucket_pair, persistent CTAs): every element gets
//         its rank among the equal tuples of its side in posting / arrival
//         order (quarters walked by one warp each with match.any peers) --
//         the receive of rank r takes the message of rank r, the MPI result
//         without wildcards;
//       - NOWILD_UNORDERED (k_bucket_pop): messages are pushed onto per-tuple
//         lists and receives pop from them -- a maximal pairing of equal
//         tuples, what the relaxation allows;
//  3. write results at the elements' snapshot positions and matched flags for
//     the queue compaction.
// A bucket larger than the on-chip capacity raises a flag; the host then runs
// the global sort-and-rank (ordered) or HBM hash-table (unordered) kernels of
// k_flat.cu for that batch instead.
#include "mm_kernels.h"
#include "mm_smem.cuh"

namespace mm {

// Bucket hash: Fibonacci (multiply-shift) hashing of the 64-bit tuple -- a
// handful of instructions instead of three Jenkins rounds, and independent of
// mm_route's owner hash (Jenkins), so the shard a rank owns still spreads over
// all buckets.  It is computed once per element (first partition pass) and
// then carried in the payload's high half.
__device__ __forceinline__ uint32_t bucket_of(uint64_t h, int nb) {
  return (uint32_t)((h * 0x9E3779B97F4A7C15ull) >> (64 - nb));
}


struct SnapRead {
  // snapshot element u: residual queue entries [0, resid), then the pending batch
  const uint64_t* q;  // residual headers (endpoint 0)
  const uint64_t* p;  // pending headers (nullptr if none)
  int64_t resid;
  __device__ __forceinline__ uint64_t hdr(int64_t u) const { return u < resid ? q[u] : p[u - resid]; }
};

// payload of a partitioned element: header word + (bucket << 32 | snapshot index)
template <bool FIRST>
struct BDigit {
  SnapRead snap;
  const uint64_t* bi;
  int nb, shift, dmask;
  __device__ __forceinline__ uint32_t operator()(int64_t k) const {
    const uint32_t b = FIRST ? bucket_of(snap.hdr(k), nb) : (uint32_t)(bi[k] >> 32);
    return (b >> shift) & (uint32_t)dmask;
  }
  // the same digit from the element's loaded payload (BMove::load)
  __device__ __forceinline__ uint32_t of_payload(int64_t, uint64_t a, uint64_t b) const {
    return ((uint32_t)(b >> 32) >> shift) & (uint32_t)dmask;
  }
};
template <bool FIRST>
struct BMove {
  SnapRead snap;
  const uint64_t* h;
  const uint64_t* bi;
  int nb;
  uint64_t* oh;
  uint64_t* obi;
  __device__ __forceinline__ void load(int64_t k, uint64_t& a, uint64_t& b) const {
    if (FIRST) {
      a = snap.hdr(k);
      b = ((uint64_t)bucket_of(a, nb) << 32) | (uint64_t)k;
    } else {
      a = h[k];
      b = bi[k];
    }
  }
  __device__ __forceinline__ void store(int64_t dst, uint64_t a, uint64_t b) const {
    oh[dst] = a;
    obi[dst] = b;
  }
};

// off[b] = first position of bucket b in the bucket-sorted array (b in 0..B).
// Four consecutive elements per thread, read as two 16-byte vectors.
__global__ void k_bucket_bounds(const uint64_t* bi, int64_t n, int nb, uint32_t* off) {
  const uint32_t B = 1u << nb;
  const int64_t nq = (n + 3) / 4;
  for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < nq; q += (int64_t)gridDim.x * blockDim.x) {
    const int64_t p0 = q * 4;
    uint64_t v[4];
    if (p0 + 4 <= n) {
      const ulonglong2 x = reinterpret_cast<const ulonglong2*>(bi + p0)[0];
      const ulonglong2 y = reinterpret_cast<const ulonglong2*>(bi + p0)[1];
      v[0] = x.x;
      v[1] = x.y;
      v[2] = y.x;
      v[3] = y.y;
    } else {
#pragma unroll
      for (int j = 0; j < 4; j++) v[j] = p0 + j < n ? bi[p0 + j] : 0ull;
    }
    uint32_t prev = p0 == 0 ? 0xFFFFFFFFu : (uint32_t)(bi[p0 - 1] >> 32);
#pragma unroll
    for (int j = 0; j < 4; j++) {
      const int64_t p = p0 + j;
      if (p >= n) break;
      const uint32_t b = (uint32_t)(v[j] >> 32);
      if (b != prev)
        for (uint32_t x = prev + 1; x <= b; x++) off[x] = (uint32_t)p;  // (prev+1 wraps to 0 at p == 0)
      if (p == n - 1)
        for (uint32_t x = b + 1; x <= B; x++) off[x] = (uint32_t)n;
      prev = b;
    }
  }
}
__global__ void k_fill_u32(uint32_t* a, int64_t n, uint32_t v) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) a[i] = v;
}

static int grid_cap(int64_t n, int threads) {
  int64_t b = (n + threads - 1) / threads;
  if (b > 148 * 32) b = 148 * 32;
  return b < 1 ? 1 : (int)b;
}

// Partition one side of the snapshot into bucket order.
static cudaError_t partition_side(const SnapRead& snap, int64_t n, int nb, uint64_t* h0, uint64_t* i0, uint64_t* h1,
                                  uint64_t* i1, uint32_t* part, uint32_t* off, uint64_t** out_h, uint64_t** out_i,
                                  cudaStream_t st) {
  const uint32_t B = 1u << nb;
  if (n == 0) {
    count_launch();
    k_fill_u32<<<grid_cap(B + 1, 256), 256, 0, st>>>(off, B + 1, 0u);
    *out_h = h0;
    *out_i = i0;
    return cudaGetLastError();
  }
  const int passes = (nb + 8) / 9;  // up to 9 bits (512 buckets) per pass
  const int dbits = (nb + passes - 1) / passes;
  uint64_t* hb[2] = {h0, h1};
  uint64_t* ib[2] = {i0, i1};
  int cur = 0;
  cudaError_t err;
  for (int p = 0; p < passes; p++) {
    const int shift = p * dbits;
    const int bits = nb - shift < dbits ? nb - shift : dbits;
    const int nbk = 1 << bits;
    if (p == 0) {
      err = partition_stable(BDigit<true>{snap, nullptr, nb, shift, nbk - 1},
                             BMove<true>{snap, nullptr, nullptr, nb, hb[cur], ib[cur]}, n, nbk, part, st);
    } else {
      err = partition_stable(BDigit<false>{snap, ib[cur], nb, shift, nbk - 1},
                             BMove<false>{snap, hb[cur], ib[cur], nb, hb[cur ^ 1], ib[cur ^ 1]}, n, nbk, part, st);
      cur ^= 1;
    }
    if (err != cudaSuccess) return err;
  }
  count_launch();
  k_bucket_bounds<<<grid_cap((n + 3) / 4, 256), 256, 0, st>>>(ib[cur], n, nb, off);
  *out_h = hb[cur];
  *out_i = ib[cur];
  return cudaGetLastError();
}

// ------------------------------------------------------------- bucket kernel
constexpr int kBucketCap = 1024;   // elements (receives + messages) per bucket on chip
constexpr int kBucketThreads = 256;
constexpr uint32_t kBucketH = 2048;  // hash slots (>= 2 * kBucketCap)
constexpr int kQ = 4;                // ordered: quarters per side, ranked by one warp each
constexpr int kPairThreads = 256;    // ordered kernel (512 measured 14 % slower)

struct BucketArgs {
  FlatArgs a;
  const uint64_t* rh;  // bucket-sorted receive headers
  const uint64_t* ri;  // (bucket << 32) | snapshot index
  const uint32_t* roff;
  const uint64_t* mh;
  const uint64_t* mi;
  const uint32_t* moff;
  uint32_t* overflow;
};

// Elements of a bucket are kept in snapshot order (the partition is stable),
// so an element's bucket position orders it among the equal tuples of its
// side.  Message tuples get dense ids through an open-addressing table of
// 32-bit entries (16-bit fingerprint | representative element; the CAS winner
// draws the id).  Every element then gets its rank among the equal tuples of
// its side in bucket order: each side is cut in kQ quarters, one warp per
// quarter walks it 32 elements at a time (match.any peers, per-tuple running
// counts), then per-tuple prefixes over the quarters complete the ranks.
// Messages are placed by (tuple, rank) after a scan of the per-tuple message
// counts, and the receive of rank r takes the message of rank r of its tuple.
// O(1) work per element (no list walks, no run-length limit), 7 barriers;
// message flags are written directly by the receive that takes the message.
struct BucketSmem {
  uint64_t hdr[kBucketCap];  // receives [0, nr), then messages [nr, nr + nm)
  uint32_t idx[kBucketCap];  // snapshot index
  union {
    struct {                     // phases A..C
      uint32_t table[kBucketH];  // tuple table
      uint16_t sid[kBucketH];    // slot -> dense tuple id (valid where table[slot] is set)
    };
    struct {                        // phases D..F
      uint16_t mstart[kBucketCap];  // tuple -> first position in msg_at
      uint16_t mtot[kBucketCap];    // tuple -> number of messages
      uint16_t msg_at[kBucketCap];  // messages grouped by tuple, in rank order
    };
  };
  uint16_t tup[kBucketCap];  // element -> slot (messages, phase B), then tuple id | kNone
  uint16_t rnk[kBucketCap];  // element -> rank among its side's equal tuples
  // qcnt[side][quarter][tuple]: running counts, then exclusive prefixes over
  // the quarters
  uint16_t qcnt[2 * kQ * kBucketCap];
  uint32_t scan_sm[kPairThreads / 32 + 1];
  uint32_t ntup;
};
static_assert(sizeof(BucketSmem) <= 44 * 1024 + 512, "five CTAs per SM");

// quarter of position x in a side of length L (boundaries q * L / kQ)
__device__ __forceinline__ uint32_t quarter_of(uint32_t x, uint32_t L) {
  return (uint32_t)(x >= L / 4) + (uint32_t)(x >= L / 2) + (uint32_t)(x >= (3 * L) / 4);
}

// Optional per-phase cycle accounting of k_bucket_pair (build with
// -DMM_PHASE_TIMING; read by mm_debug_bucket_cycles): thread 0 adds clock64
// deltas per phase, slot 15 counts buckets.
#ifdef MM_PHASE_TIMING
__device__ unsigned long long g_bucket_cycles[16];
#define MM_BPHASE(n)                                                        \
  do {                                                                     \
    if (threadIdx.x == 0) {                                                \
      const long long _t = clock64();                                      \
      atomicAdd(&g_bucket_cycles[n], (unsigned long long)(_t - t_bphase)); \
      t_bphase = _t;                                                       \
    }                                                                      \
  } while (0)
#else
#define MM_BPHASE(n) \
  do {               \
  } while (0)
#endif

__global__ void __launch_bounds__(kPairThreads, 5) k_bucket_pair(BucketArgs ba, uint32_t nbk) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  BucketSmem& sm = *reinterpret_cast<BucketSmem*>(smem_raw);
  constexpr int NT = kPairThreads;
  constexpr int PER = kBucketCap / NT;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const FlatArgs& a = ba.a;
  const int64_t rres = a.R.q_len[0], rpb = a.R.pend_begin(0);
  const int64_t mres = a.M.q_len[0], mpb = a.M.pend_begin(0);
  constexpr uint32_t hmask = kBucketH - 1;
  // Persistent: buckets blockIdx.x, + gridDim.x, ...; the next bucket's
  // elements are loaded into registers while the current one is matched.
  uint64_t hv[PER];
  uint32_t iv[PER];
  auto fetch = [&](uint32_t bb, uint32_t& fr0, uint32_t& fnr, uint32_t& fm0, uint32_t& fnm) {
    fr0 = fnr = fm0 = fnm = 0;
    if (bb < nbk) {
      fr0 = ba.roff[bb];
      fnr = ba.roff[bb + 1] - fr0;
      fm0 = ba.moff[bb];
      fnm = ba.moff[bb + 1] - fm0;
    }
    const bool fits = fnr + fnm <= (uint32_t)kBucketCap;
#pragma unroll
    for (int u = 0; u < PER; u++) {
      const uint32_t e = tid + u * NT;
      hv[u] = 0;
      iv[u] = 0;
      if (fits && e < fnr) {
        hv[u] = ba.rh[fr0 + e];
        iv[u] = (uint32_t)ba.ri[fr0 + e];
      } else if (fits && e < fnr + fnm) {
        hv[u] = ba.mh[fm0 + e - fnr];
        iv[u] = (uint32_t)ba.mi[fm0 + e - fnr];
      }
    }
  };
  uint32_t xr0, xnr, xm0, xnm;  // bounds of the bucket held in hv / iv
#ifdef MM_PHASE_TIMING
  long long t_bphase = clock64();
#endif
  fetch(blockIdx.x, xr0, xnr, xm0, xnm);
  for (uint32_t b = blockIdx.x; b < nbk; b += gridDim.x) {
    __syncthreads();  // the previous bucket is done with shared memory
    MM_BPHASE(0);
    const uint32_t r0 = xr0, nr = xnr, m0 = xm0, nm = xnm;
    const uint32_t n = nr + nm;
    if (n == 0 || n > (uint32_t)kBucketCap) {  // uniform across the CTA
      if (n > (uint32_t)kBucketCap && tid == 0) atomicOr(ba.overflow, 1u);
      fetch(b + gridDim.x, xr0, xnr, xm0, xnm);
      continue;
    }
    // A: registers to shared memory, clear the tables, prefetch the next bucket
#pragma unroll
    for (int u = 0; u < PER; u++) {
      const uint32_t e = tid + u * NT;
      if (e < n) {
        sm.hdr[e] = hv[u];
        sm.idx[e] = iv[u];
      }
    }
    for (uint32_t s = tid; s < kBucketH / 4; s += NT) reinterpret_cast<uint4*>(sm.table)[s] = make_uint4(~0u, ~0u, ~0u, ~0u);
    if (tid == 0) sm.ntup = 0;
    // message flags start at 0; phase F sets the matched ones (the barriers
    // in between order the two stores)
    for (uint32_t x = tid; x < nm; x += NT) a.mflag[m0 + x] = 0;
    fetch(b + gridDim.x, xr0, xnr, xm0, xnm);
    __syncthreads();
    MM_BPHASE(1);
    // B: message tuples into the table; the CAS winner draws the dense id
    for (uint32_t e = nr + tid; e < n; e += NT) {
      const uint64_t h = sm.hdr[e];
      const uint64_t p = h * 0xD6E8FEB86659FD93ull;
      uint32_t s = (uint32_t)(p >> 40) & hmask;
      const uint32_t fp = (uint32_t)(p >> 24) & 0xFFFFu;
      while (true) {
        uint32_t o = sm.table[s];
        if (o == 0xFFFFFFFFu) {
          o = atomicCAS(&sm.table[s], 0xFFFFFFFFu, (fp << 16) | e);  // representative's header is in smem already
          if (o == 0xFFFFFFFFu) {
            sm.sid[s] = (uint16_t)atomicAdd(&sm.ntup, 1u);
            break;
          }
        }
        if ((o >> 16) == fp && sm.hdr[o & 0xFFFFu] == h) break;
        s = (s + 1) & hmask;
      }
      sm.tup[e] = (uint16_t)s;
    }
    __syncthreads();
    MM_BPHASE(2);
    const uint32_t T = sm.ntup;
    // C1: tuple ids of every element (receives look theirs up); the
    // per-quarter running counts of the T tuples cleared
    for (uint32_t e = tid; e < n; e += NT) {
      uint32_t id = kNone;
      if (e >= nr) {
        id = sm.sid[sm.tup[e]];
      } else {
        const uint64_t h = sm.hdr[e];
        const uint64_t p = h * 0xD6E8FEB86659FD93ull;
        uint32_t s = (uint32_t)(p >> 40) & hmask;
        const uint32_t fp = (uint32_t)(p >> 24) & 0xFFFFu;
        while (true) {
          const uint32_t o = sm.table[s];
          if (o == 0xFFFFFFFFu) break;
          if ((o >> 16) == fp && sm.hdr[o & 0xFFFFu] == h) {
            id = sm.sid[s];
            break;
          }
          s = (s + 1) & hmask;
        }
      }
      sm.tup[e] = (uint16_t)id;
    }
    {
      const uint32_t T8 = (T + 7) / 8;  // 16-byte words per row
      for (uint32_t x = tid; x < 2 * kQ * T8; x += NT)
        reinterpret_cast<uint4*>(&sm.qcnt[(x / T8) * kBucketCap])[x % T8] = make_uint4(0u, 0u, 0u, 0u);
    }
    __syncthreads();
    // C2: ranks within the side -- one warp per quarter walks it 32 elements
    // at a time (match.any peers, per-tuple running counts)
    if (warp < 2 * kQ) {
      const uint32_t side = warp < kQ ? 1u : 0u, q = warp & (kQ - 1);
      uint16_t* run = &sm.qcnt[(side * kQ + q) * kBucketCap];
      const uint32_t L = side ? nm : nr, base = side ? nr : 0u;
      const uint32_t lo = base + (q * L) / kQ, hi = base + ((q + 1) * L) / kQ;
      const uint32_t lt = lanemask_lt();
      for (uint32_t c = lo; c < hi; c += 32) {
        const uint32_t e = c + lane;
        const uint32_t id = e < hi ? sm.tup[e] : kNone;
        const bool has = id != kNone;
        const uint32_t peers = __match_any_sync(kFull, has ? id : 0x10000u + lane);
        const uint32_t before = has ? run[id] : 0u;
        __syncwarp();
        if (has && (peers >> lane) == 1u) run[id] = (uint16_t)(before + __popc(peers));  // highest peer publishes
        if (e < hi) sm.rnk[e] = (uint16_t)(before + __popc(peers & lt));
        __syncwarp();
      }
    }
    __syncthreads();
    MM_BPHASE(3);
    // D: per tuple -- prefixes over the quarters, message totals, and their
    // scan (tuples TPT * tid .. TPT * tid + TPT - 1)
    {
      constexpr int TPT = kBucketCap / NT;  // tuples per thread
      uint32_t tot[TPT], sum = 0;
#pragma unroll
      for (int j = 0; j < TPT; j++) {
        const uint32_t t = TPT * tid + j;
        tot[j] = 0;
        if (t < T) {
#pragma unroll
          for (int side = 0; side < 2; side++) {
            uint32_t acc = 0;
#pragma unroll
            for (int q = 0; q < kQ; q++) {
              uint16_t* c = &sm.qcnt[(side * kQ + q) * kBucketCap + t];
              const uint32_t v = *c;
              *c = (uint16_t)acc;
              acc += v;
            }
            if (side) tot[j] = acc;
          }
        }
        sum += tot[j];
      }
      uint32_t all;
      uint32_t ex = block_excl_scan<uint32_t>(sum, sm.scan_sm, &all);
#pragma unroll
      for (int j = 0; j < TPT; j++) {
        const uint32_t t = TPT * tid + j;
        if (t < T) {
          sm.mstart[t] = (uint16_t)ex;
          sm.mtot[t] = (uint16_t)tot[j];
        }
        ex += tot[j];
      }
    }
    __syncthreads();
    MM_BPHASE(4);
    // E: full ranks; messages placed by (tuple, rank)
    for (uint32_t e = tid; e < n; e += NT) {
      const uint32_t id = sm.tup[e];
      if (id == kNone) continue;
      const uint32_t side = e >= nr ? 1u : 0u;
      const uint32_t q = side ? quarter_of(e - nr, nm) : quarter_of(e, nr);
      const uint32_t r = sm.rnk[e] + sm.qcnt[(side * kQ + q) * kBucketCap + id];
      if (!side) sm.rnk[e] = (uint16_t)r;
      if (e >= nr) sm.msg_at[sm.mstart[id] + r] = (uint16_t)e;
    }
    __syncthreads();
    MM_BPHASE(5);
    // F: receives take the message of equal rank
    uint32_t nmatch = 0;
    for (uint32_t e = tid; e < nr; e += NT) {
      const uint32_t id = sm.tup[e];
      uint32_t j = kNone;
      if (id != kNone) {
        const uint32_t r = sm.rnk[e];
        if (r < sm.mtot[id]) j = sm.msg_at[sm.mstart[id] + r];
      }
      int64_t mc = MM_NO_MATCH;
      if (j != kNone) {
        a.mflag[m0 + (j - nr)] = 1;
        mc = a.M.cookie(0, sm.idx[j], mres, mpb);
        nmatch++;
      }
      a.out_rc[r0 + e] = a.R.cookie(0, sm.idx[e], rres, rpb);
      a.out_mc[r0 + e] = mc;
      a.rflag[r0 + e] = j != kNone ? 1 : 0;
    }
    for (int o = 16; o; o >>= 1) nmatch += __shfl_xor_sync(kFull, nmatch, o);
    if (lane == 0 && nmatch) atomicAdd(a.n_matched, (unsigned long long)nmatch);
    MM_BPHASE(6);
#ifdef MM_PHASE_TIMING
    if (threadIdx.x == 0) atomicAdd(&g_bucket_cycles[15], 1ull);
#endif
  }
}

#ifndef MM_POP_MIN_BLOCKS
#define MM_POP_MIN_BLOCKS 6  // resident CTAs per SM the register budget must allow (28.8 KB smem allows 7)
#endif
// NOWILD_UNORDERED: messages pushed onto per-tuple lists, receives pop from
// them (lock-free, pops only in that phase: no ABA) -- any maximal pairing of
// equal tuples; 3 barriers, message flags written by the popping receive.
struct PopSmem {
  uint64_t hdr[kBucketCap];               // receives [0, nr), then messages [nr, nr + nm)
  uint32_t idx[kBucketCap];               // snapshot index
  uint32_t table[kBucketH];               // tuple table
  uint16_t mhead[kBucketH];               // per slot: message list
  uint16_t next[kBucketCap];              // list links
  uint16_t slot[kBucketCap];              // receive -> slot | kNone
};

__global__ void __launch_bounds__(kBucketThreads, MM_POP_MIN_BLOCKS) k_bucket_pop(BucketArgs ba, uint32_t nbk) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  PopSmem& sm = *reinterpret_cast<PopSmem*>(smem_raw);
  constexpr int NT = kBucketThreads;
  constexpr int PER = kBucketCap / NT;
  const int tid = threadIdx.x, lane = tid & 31;
  const FlatArgs& a = ba.a;
  const int64_t rres = a.R.q_len[0], rpb = a.R.pend_begin(0);
  const int64_t mres = a.M.q_len[0], mpb = a.M.pend_begin(0);
  constexpr uint32_t hmask = kBucketH - 1;
  // Persistent: buckets blockIdx.x, + gridDim.x, ...; the next bucket's
  // elements are loaded into registers while the current one is matched.
  uint64_t hv[PER];
  uint32_t iv[PER];
  auto fetch = [&](uint32_t bb, uint32_t& fr0, uint32_t& fnr, uint32_t& fm0, uint32_t& fnm) {
    fr0 = fnr = fm0 = fnm = 0;
    if (bb < nbk) {
      fr0 = ba.roff[bb];
      fnr = ba.roff[bb + 1] - fr0;
      fm0 = ba.moff[bb];
      fnm = ba.moff[bb + 1] - fm0;
    }
    const bool fits = fnr + fnm <= (uint32_t)kBucketCap;
#pragma unroll
    for (int u = 0; u < PER; u++) {
      const uint32_t e = tid + u * NT;
      hv[u] = 0;
      iv[u] = 0;
      if (fits && e < fnr) {
        hv[u] = ba.rh[fr0 + e];
        iv[u] = (uint32_t)ba.ri[fr0 + e];
      } else if (fits && e < fnr + fnm) {
        hv[u] = ba.mh[fm0 + e - fnr];
        iv[u] = (uint32_t)ba.mi[fm0 + e - fnr];
      }
    }
  };
  uint32_t xr0, xnr, xm0, xnm;  // bounds of the bucket held in hv / iv
  fetch(blockIdx.x, xr0, xnr, xm0, xnm);
  for (uint32_t b = blockIdx.x; b < nbk; b += gridDim.x) {
    __syncthreads();  // the previous bucket is done with shared memory
    const uint32_t r0 = xr0, nr = xnr, m0 = xm0, nm = xnm;
    const uint32_t n = nr + nm;
    if (n == 0 || n > (uint32_t)kBucketCap) {  // uniform across the CTA
      if (n > (uint32_t)kBucketCap && tid == 0) atomicOr(ba.overflow, 1u);
      fetch(b + gridDim.x, xr0, xnr, xm0, xnm);
      continue;
    }
    // registers to shared memory, clear the tables, prefetch the next bucket
    {
#pragma unroll
      for (int u = 0; u < PER; u++) {
        const uint32_t e = tid + u * NT;
        if (e < n) {
          sm.hdr[e] = hv[u];
          sm.idx[e] = iv[u];
        }
      }
      for (uint32_t s = tid; s < kBucketH / 4; s += NT) reinterpret_cast<uint4*>(sm.table)[s] = make_uint4(~0u, ~0u, ~0u, ~0u);
      for (uint32_t s = tid; s < kBucketH / 8; s += NT) reinterpret_cast<uint4*>(sm.mhead)[s] = make_uint4(~0u, ~0u, ~0u, ~0u);
      // message flags start at 0; the receive that pops a message sets its
      // flag (the barriers in between order the two stores)
      for (uint32_t x = tid; x < nm; x += NT) a.mflag[m0 + x] = 0;
      fetch(b + gridDim.x, xr0, xnr, xm0, xnm);
    }
    __syncthreads();
    // messages: find or open the tuple's slot, push onto its message list
    for (uint32_t e = nr + tid; e < n; e += NT) {
      const uint64_t h = sm.hdr[e];
      const uint64_t p = h * 0xD6E8FEB86659FD93ull;
      uint32_t s = (uint32_t)(p >> 40) & hmask;
      const uint32_t fp = (uint32_t)(p >> 24) & 0xFFFFu;
      while (true) {
        uint32_t o = sm.table[s];
        if (o == 0xFFFFFFFFu) {
          o = atomicCAS(&sm.table[s], 0xFFFFFFFFu, (fp << 16) | e);  // representative's header is in smem already
          if (o == 0xFFFFFFFFu) break;
        }
        if ((o >> 16) == fp && sm.hdr[o & 0xFFFFu] == h) break;
        s = (s + 1) & hmask;
      }
      sm.next[e] = exch16(&sm.mhead[s], (uint16_t)e);
    }
    __syncthreads();
    // receives: look the tuple up
    for (uint32_t e = tid; e < nr; e += NT) {
      const uint64_t h = sm.hdr[e];
      const uint64_t p = h * 0xD6E8FEB86659FD93ull;
      uint32_t s = (uint32_t)(p >> 40) & hmask;
      const uint32_t fp = (uint32_t)(p >> 24) & 0xFFFFu;
      uint32_t found = kNone;
      while (true) {
        const uint32_t o = sm.table[s];
        if (o == 0xFFFFFFFFu) break;
        if ((o >> 16) == fp && sm.hdr[o & 0xFFFFu] == h) {
          found = s;
          break;
        }
        s = (s + 1) & hmask;
      }
      sm.slot[e] = (uint16_t)found;
    }
    __syncthreads();
    // receives take any message of their tuple (pop from the list)
    uint32_t nmatch = 0;
    for (uint32_t e = tid; e < nr; e += NT) {
      const uint32_t s = sm.slot[e];
      uint32_t j = kNone;
      if (s != kNone) {
        uint32_t hd = sm.mhead[s];
        while (hd != kNone) {  // pops only in this phase: no ABA
          const uint32_t got = cas16(&sm.mhead[s], (uint16_t)hd, sm.next[hd]);
          if (got == hd) {
            j = hd;
            break;
          }
          hd = got;
        }
      }
      int64_t mc = MM_NO_MATCH;
      if (j != kNone) {
        a.mflag[m0 + (j - nr)] = 1;
        mc = a.M.cookie(0, sm.idx[j], mres, mpb);
        nmatch++;
      }
      a.out_rc[r0 + e] = a.R.cookie(0, sm.idx[e], rres, rpb);
      a.out_mc[r0 + e] = mc;
      a.rflag[r0 + e] = j != kNone ? 1 : 0;
    }
    for (int o = 16; o; o >>= 1) nmatch += __shfl_xor_sync(kFull, nmatch, o);
    if (lane == 0 && nmatch) atomicAdd(a.n_matched, (unsigned long long)nmatch);
  }
}

// ~512 elements per bucket on average (capacity 1024: a bucket overflows
// only for heavily repeated tuples)
int64_t bucket_bits_for(int64_t n) {
  int nb = 1;
  while (nb < 27 && ((int64_t)1 << nb) * 512 < n) nb++;
  return nb;
}

// persistent grid: every resident CTA slot of the chip, at most one per bucket
template <auto KERNEL>
static uint32_t bucket_grid(int threads, size_t smem, uint32_t B) {
  const uint32_t g = (uint32_t)resident_ctas<KERNEL>(threads, smem);
  return g < B ? g : B;
}

cudaError_t run_bucketed(const FlatArgs& a, bool ordered, BucketScratch& s, cudaStream_t st) {
  const int nb = (int)bucket_bits_for(a.nr + a.nm);
  const uint32_t B = 1u << nb;
  // single endpoint: the pending batch starts at 0
  SnapRead rs{a.R.q_hdr, a.R.p_hdr, s.rres}, ms{a.M.q_hdr, a.M.p_hdr, s.mres};
  uint64_t *rh, *mh;
  uint64_t *ri, *mi;
  // the two sides are independent until the bucket kernel: the messages are
  // partitioned on a second stream (their small scan kernels and launch gaps
  // overlap the receives' passes)
  cudaStream_t mst = st;
  cudaError_t err;
  if (s.side_st) {
    if ((err = cudaEventRecord(s.ev_fork, st)) != cudaSuccess) return err;
    if ((err = cudaStreamWaitEvent(s.side_st, s.ev_fork, 0)) != cudaSuccess) return err;
    mst = s.side_st;
  }
  err = partition_side(rs, a.nr, nb, s.h[0], s.i[0], s.h[1], s.i[1], s.part, s.roff, &rh, &ri, st);
  if (err != cudaSuccess) return err;
  err = partition_side(ms, a.nm, nb, s.h[2], s.i[2], s.h[3], s.i[3], s.side_st ? s.part2 : s.part, s.moff, &mh, &mi,
                       mst);
  if (err != cudaSuccess) return err;
  if (s.side_st) {
    if ((err = cudaEventRecord(s.ev_join, s.side_st)) != cudaSuccess) return err;
    if ((err = cudaStreamWaitEvent(st, s.ev_join, 0)) != cudaSuccess) return err;
  }
  if ((err = cudaMemsetAsync(s.overflow, 0, 4, st)) != cudaSuccess) return err;
  s.rh_sorted = rh;
  s.ri_sorted = ri;
  s.mh_sorted = mh;
  s.mi_sorted = mi;
  BucketArgs ba{a, rh, ri, s.roff, mh, mi, s.moff, s.overflow};
  if (ordered) {
    const size_t smem = sizeof(BucketSmem);
    err = ensure_dyn_smem<k_bucket_pair>(smem);
    if (err != cudaSuccess) return err;
    count_launch();
    k_bucket_pair<<<bucket_grid<k_bucket_pair>(kPairThreads, smem, B), kPairThreads, smem, st>>>(ba, B);
  } else {
    const size_t smem = sizeof(PopSmem);
    err = ensure_dyn_smem<k_bucket_pop>(smem);
    if (err != cudaSuccess) return err;
    count_launch();
    k_bucket_pop<<<bucket_grid<k_bucket_pop>(kBucketThreads, smem, B), kBucketThreads, smem, st>>>(ba, B);
  }
  return cudaGetLastError();
}

// Residual queue from the bucket-sorted side: survivors keep bucket order
// (hence per-tuple order).
struct SortedUnmatched {
  const uint8_t* matched;
  __device__ __forceinline__ uint32_t operator()(int64_t p) const { return matched[p] ? 0u : 1u; }
};
struct SortedCompactOut {
  Side S;
  int64_t resid;
  const uint64_t* h;
  const uint64_t* ix;
  int64_t n;
  uint64_t* q_h;
  int64_t* q_c;
  int32_t* q_len;
  __device__ __forceinline__ void operator()(int64_t p, uint32_t ex, uint32_t v) const {
    if (v) {
      q_h[ex] = h[p];
      q_c[ex] = S.cookie(0, (uint32_t)ix[p], resid, 0);
    }
    if (p == n - 1) *q_len = (int32_t)(ex + v);
  }
};
__global__ void k_set_len0(int32_t* q_len) { *q_len = 0; }

cudaError_t run_compact_sorted(const Side& S, int64_t resid, int64_t n, const uint64_t* h, const uint64_t* ix,
                               const uint8_t* matched, uint64_t* q_h, int64_t* q_c, int32_t* q_len, uint32_t* scan,
                               cudaStream_t st) {
  if (n == 0) {
    count_launch();
    k_set_len0<<<1, 1, 0, st>>>(q_len);
    return cudaGetLastError();
  }
  return scan_apply<uint32_t>(SortedUnmatched{matched}, n, scan, SortedCompactOut{S, resid, h, ix, n, q_h, q_c, q_len},
                              st);
}

int64_t bucket_scratch_elems(int64_t n) { return ((int64_t)1 << bucket_bits_for(n)) + 1; }

}  // namespace mm

#ifdef MM_PHASE_TIMING
extern "C" int mm_debug_bucket_cycles(unsigned long long* out, int reset) {
  cudaDeviceSynchronize();
  if (cudaMemcpyFromSymbol(out, mm::g_bucket_cycles, sizeof(unsigned long long) * 16) != cudaSuccess) return 2;
  if (reset) {
    unsigned long long z[16] = {0};
    cudaMemcpyToSymbol(mm::g_bucket_cycles, z, sizeof(z));
  }
  return 0;
}
#endif
