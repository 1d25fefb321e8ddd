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
//     go into a lock-free open-addressing hash table (16-bit CAS), receives
//     look their tuple up, and each element gets its rank among the equal
//     tuples of its side:
//       - NOWILD_ORDERED: ranks in posting / arrival order (warp-ordered
//         placement, quarters in parallel) -- the n-th receive of a tuple takes
//         the n-th message of it, the MPI result without wildcards;
//       - NOWILD_UNORDERED: ranks from shared-memory atomics, any order -- a
//         maximal pairing of equal tuples, what the relaxation allows;
//     the receive of rank r pairs with the message of rank r;
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
constexpr uint32_t kMaxRun = 64;     // ordered: longest run of one tuple walked on chip

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
// side.  Tuples are found through an open-addressing table of 32-bit entries
// (16-bit fingerprint | representative element); the elements of a tuple form
// singly linked lists per side, pushed with one atomic exchange each.
template <bool ORDERED>
struct BucketSmem {
  uint64_t hdr[kBucketCap];               // receives [0, nr), then messages [nr, nr + nm)
  uint32_t idx[kBucketCap];               // snapshot index
  uint32_t table[kBucketH];               // tuple table
  uint16_t mhead[kBucketH];               // per slot: message list
  uint16_t rhead[ORDERED ? kBucketH : 2];  // per slot: receive list (ordered)
  uint16_t next[kBucketCap];              // list links
  uint16_t slot[kBucketCap];              // receive -> slot | kNone
  uint16_t rank[ORDERED ? kBucketCap : 2];  // message rank among its tuple's messages
  uint32_t matched[kBucketCap / 32];      // message matched bits (by message offset)
};

template <bool ORDERED>
__global__ void __launch_bounds__(kBucketThreads) k_bucket_pair(BucketArgs ba) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  BucketSmem<ORDERED>& sm = *reinterpret_cast<BucketSmem<ORDERED>*>(smem_raw);
  constexpr int NT = kBucketThreads;
  const int tid = threadIdx.x, lane = tid & 31;
  const FlatArgs& a = ba.a;
  const int b = blockIdx.x;
  const uint32_t r0 = ba.roff[b], nr = ba.roff[b + 1] - r0;
  const uint32_t m0 = ba.moff[b], nm = ba.moff[b + 1] - m0;
  if (nr + nm == 0) return;
  if (nr + nm > (uint32_t)kBucketCap) {
    if (tid == 0) atomicOr(ba.overflow, 1u);
    return;
  }
  const uint32_t n = nr + nm;
  const int64_t rres = a.R.q_len[0], rpb = a.R.pend_begin(0);
  const int64_t mres = a.M.q_len[0], mpb = a.M.pend_begin(0);
  constexpr uint32_t hmask = kBucketH - 1;
  // load (all loads of a thread in flight), clear the tables
  {
    constexpr int PER = kBucketCap / NT;
    uint64_t hv[PER], iv[PER];
#pragma unroll
    for (int u = 0; u < PER; u++) {
      const uint32_t e = tid + u * NT;
      hv[u] = 0;
      iv[u] = 0;
      if (e < nr) {
        hv[u] = ba.rh[r0 + e];
        iv[u] = ba.ri[r0 + e];
      } else if (e < n) {
        hv[u] = ba.mh[m0 + e - nr];
        iv[u] = ba.mi[m0 + e - nr];
      }
    }
    for (uint32_t s = tid; s < kBucketH / 4; s += NT) reinterpret_cast<uint4*>(sm.table)[s] = make_uint4(~0u, ~0u, ~0u, ~0u);
    for (uint32_t s = tid; s < kBucketH / 8; s += NT) reinterpret_cast<uint4*>(sm.mhead)[s] = make_uint4(~0u, ~0u, ~0u, ~0u);
    if (ORDERED)
      for (uint32_t s = tid; s < kBucketH / 8; s += NT) reinterpret_cast<uint4*>(sm.rhead)[s] = make_uint4(~0u, ~0u, ~0u, ~0u);
    for (uint32_t s = tid; s < kBucketCap / 32; s += NT) sm.matched[s] = 0u;
#pragma unroll
    for (int u = 0; u < PER; u++) {
      const uint32_t e = tid + u * NT;
      if (e < n) {
        sm.hdr[e] = hv[u];
        sm.idx[e] = (uint32_t)iv[u];
      }
    }
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
  // receives: look the tuple up (ordered: push onto its receive list)
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
    if (ORDERED && found != kNone) sm.next[e] = exch16(&sm.rhead[found], (uint16_t)e);
  }
  if (ORDERED) {
    // message ranks: earlier messages of the same tuple have smaller positions
    for (uint32_t e = nr + tid; e < n; e += NT) {
      const uint64_t h = sm.hdr[e];
      const uint64_t p = h * 0xD6E8FEB86659FD93ull;
      uint32_t s = (uint32_t)(p >> 40) & hmask;
      const uint32_t fp = (uint32_t)(p >> 24) & 0xFFFFu;
      while (true) {
        const uint32_t o = sm.table[s];
        if ((o >> 16) == fp && sm.hdr[o & 0xFFFFu] == h) break;
        s = (s + 1) & hmask;
      }
      uint32_t r = 0, len = 0;
      for (uint32_t x = sm.mhead[s]; x != kNone && len <= kMaxRun; x = sm.next[x], len++) r += x < e;
      if (len > kMaxRun) atomicOr(ba.overflow, 1u);  // a tuple too long to rank by walking
      sm.rank[e] = (uint16_t)r;
    }
  }
  __syncthreads();
  // receives take their message: ordered -- the message of equal rank;
  // unordered -- any message of the tuple (pop from the list)
  uint32_t nmatch = 0;
  for (uint32_t e = tid; e < nr; e += NT) {
    const uint32_t s = sm.slot[e];
    uint32_t j = kNone;
    if (s != kNone) {
      if (ORDERED) {
        uint32_t r = 0, len = 0;
        for (uint32_t x = sm.rhead[s]; x != kNone && len <= kMaxRun; x = sm.next[x], len++) r += x < e;
        if (len > kMaxRun) atomicOr(ba.overflow, 1u);
        for (uint32_t x = sm.mhead[s]; x != kNone; x = sm.next[x])
          if (sm.rank[x] == r) {
            j = x;
            break;
          }
      } else {
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
    }
    int64_t mc = MM_NO_MATCH;
    if (j != kNone) {
      atomicOr(&sm.matched[(j - nr) >> 5], 1u << ((j - nr) & 31));
      mc = a.M.cookie(0, sm.idx[j], mres, mpb);
      nmatch++;
    }
    a.out_rc[r0 + e] = a.R.cookie(0, sm.idx[e], rres, rpb);
    a.out_mc[r0 + e] = mc;
    a.rflag[r0 + e] = j != kNone ? 1 : 0;
  }
  for (int o = 16; o; o >>= 1) nmatch += __shfl_xor_sync(kFull, nmatch, o);
  if (lane == 0 && nmatch) atomicAdd(a.n_matched, (unsigned long long)nmatch);
  __syncthreads();
  for (uint32_t x = tid; x < nm; x += NT) a.mflag[m0 + x] = (sm.matched[x >> 5] >> (x & 31)) & 1u;
}

// ~512 elements per bucket on average (capacity 1024: a bucket overflows
// only for heavily repeated tuples)
int64_t bucket_bits_for(int64_t n) {
  int nb = 1;
  while (nb < 27 && ((int64_t)1 << nb) * 512 < n) nb++;
  return nb;
}

cudaError_t run_bucketed(const FlatArgs& a, bool ordered, BucketScratch& s, cudaStream_t st) {
  const int nb = (int)bucket_bits_for(a.nr + a.nm);
  const uint32_t B = 1u << nb;
  // single endpoint: the pending batch starts at 0
  SnapRead rs{a.R.q_hdr, a.R.p_hdr, s.rres}, ms{a.M.q_hdr, a.M.p_hdr, s.mres};
  uint64_t *rh, *mh;
  uint64_t *ri, *mi;
  cudaError_t err = partition_side(rs, a.nr, nb, s.h[0], s.i[0], s.h[1], s.i[1], s.part, s.roff, &rh, &ri, st);
  if (err != cudaSuccess) return err;
  err = partition_side(ms, a.nm, nb, s.h[2], s.i[2], s.h[3], s.i[3], s.part, s.moff, &mh, &mi, st);
  if (err != cudaSuccess) return err;
  if ((err = cudaMemsetAsync(s.overflow, 0, 4, st)) != cudaSuccess) return err;
  s.rh_sorted = rh;
  s.ri_sorted = ri;
  s.mh_sorted = mh;
  s.mi_sorted = mi;
  BucketArgs ba{a, rh, ri, s.roff, mh, mi, s.moff, s.overflow};
  if (ordered) {
    const size_t smem = sizeof(BucketSmem<true>);
    err = cudaFuncSetAttribute(k_bucket_pair<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (err != cudaSuccess) return err;
    count_launch();
    k_bucket_pair<true><<<B, kBucketThreads, smem, st>>>(ba);
  } else {
    const size_t smem = sizeof(BucketSmem<false>);
    err = cudaFuncSetAttribute(k_bucket_pair<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (err != cudaSuccess) return err;
    count_launch();
    k_bucket_pair<false><<<B, kBucketThreads, smem, st>>>(ba);
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
