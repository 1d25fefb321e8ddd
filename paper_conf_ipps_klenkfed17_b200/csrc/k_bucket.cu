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
  Side S;
  int64_t resid, pb;
  __device__ __forceinline__ uint64_t hdr(int64_t u) const { return S.hdr(0, u, resid, pb); }
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

template <bool ORDERED>
struct BucketSmem {
  uint64_t hdr[kBucketCap];      // receives [0, nr), then messages [nr, nr + nm)
  uint32_t idx[kBucketCap];      // snapshot index
  uint16_t key[kBucketCap];      // tuple id | kNone
  uint16_t rank[kBucketCap];     // rank among the equal tuples of the element's side
  uint16_t table[kBucketH];      // slot -> representative message (element index)
  uint16_t cnt_m[kBucketCap];    // messages per tuple
  uint16_t start_m[kBucketCap];  // start of the tuple in by_key
  uint16_t cnt_r[kBucketCap];    // receives per tuple
  uint16_t by_key[kBucketCap];   // messages grouped by tuple, in rank order (element index)
  uint16_t pcnt[ORDERED ? 4 : 2][kBucketCap];  // per-half counts / running ranks (msgs, then receives)
  uint32_t scan[kBucketThreads / 32 + 1];
  uint32_t K;
  uint32_t matched;
};

template <bool ORDERED>
__global__ void __launch_bounds__(kBucketThreads) k_bucket_pair(BucketArgs ba) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  BucketSmem<ORDERED>& sm = *reinterpret_cast<BucketSmem<ORDERED>*>(smem_raw);
  constexpr int QN = ORDERED ? 2 : 1;  // ordered: each side placed in two halves by two warps
  constexpr int RROW = QN;             // first pcnt row of the receive side
  constexpr int NT = kBucketThreads;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t lt = lanemask_lt();
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
  const uint32_t hmask = kBucketH - 1;
  for (uint32_t e = tid; e < n; e += NT) {
    if (e < nr) {
      sm.hdr[e] = ba.rh[r0 + e];
      sm.idx[e] = (uint32_t)ba.ri[r0 + e];
    } else {
      sm.hdr[e] = ba.mh[m0 + e - nr];
      sm.idx[e] = (uint32_t)ba.mi[m0 + e - nr];
    }
  }
  for (uint32_t s = tid; s < kBucketH / 2; s += NT) reinterpret_cast<uint32_t*>(sm.table)[s] = 0xFFFFFFFFu;
  if (tid == 0) {
    sm.matched = 0;
    sm.K = 0;
  }
  __syncthreads();
  // message tuples into the hash table (slot -> representative element); the
  // CAS winner takes the next dense id and records it in rank[representative]
  // (rank is only filled later, by the ranking step)
  for (uint32_t e = nr + tid; e < n; e += NT) {
    const uint64_t h = sm.hdr[e];
    uint32_t s = slot_hash(h) & hmask;
    while (true) {
      uint16_t o = sm.table[s];
      if (o == kEmpty16) {
        o = cas16(&sm.table[s], kEmpty16, (uint16_t)e);
        if (o == kEmpty16) {
          const uint32_t id = atomicAdd(&sm.K, 1u);
          sm.rank[e] = (uint16_t)id;
#pragma unroll
          for (int q = 0; q < 2 * QN; q++) sm.pcnt[q][id] = 0;
          o = (uint16_t)e;
          break;
        }
      }
      if (sm.hdr[o] == h) break;
      s = (s + 1) & hmask;
    }
    sm.key[e] = (uint16_t)(s);  // slot for now
  }
  __syncthreads();
  const uint32_t K = sm.K;
  // tuple ids; per-half counts (ordered) or plain counts (unordered)
  for (uint32_t e = tid; e < n; e += NT) {
    uint16_t k;
    const bool is_msg = e >= nr;
    if (is_msg) {
      k = sm.rank[sm.table[sm.key[e]]];
    } else {
      const uint64_t h = sm.hdr[e];
      uint32_t s = slot_hash(h) & hmask;
      k = kNone;
      while (true) {
        const uint16_t o = sm.table[s];
        if (o == kEmpty16) break;
        if (sm.hdr[o] == h) {
          k = sm.rank[o];
          break;
        }
        s = (s + 1) & hmask;
      }
    }
    sm.key[e] = k;
    if (k != kNone) {
      const uint32_t side_n = is_msg ? nm : nr, x = is_msg ? e - nr : e;
      const uint32_t q = ORDERED ? (uint32_t)(((uint64_t)x * QN) / side_n) : 0u;
      inc16(&sm.pcnt[(is_msg ? 0 : RROW) + q][k]);
    }
  }
  __syncthreads();
  {  // per tuple: quarter prefixes, totals, message list starts
    const uint32_t per = (K + NT - 1) / NT;
    const uint32_t k0 = min(K, tid * per), k1 = min(K, k0 + per);
    uint32_t c = 0;
    for (uint32_t k = k0; k < k1; k++) {
      uint32_t rm = 0, rr = 0;
#pragma unroll
      for (int q = 0; q < QN; q++) {
        const uint32_t x = sm.pcnt[q][k], y = sm.pcnt[RROW + q][k];
        sm.pcnt[q][k] = (uint16_t)rm;
        sm.pcnt[RROW + q][k] = (uint16_t)rr;
        rm += x;
        rr += y;
      }
      sm.cnt_m[k] = (uint16_t)rm;
      sm.cnt_r[k] = (uint16_t)rr;
      c += rm;
    }
    uint32_t tot;
    uint32_t st = block_excl_scan<uint32_t>(c, sm.scan, &tot);
    for (uint32_t k = k0; k < k1; k++) {
      sm.start_m[k] = (uint16_t)st;
      st += sm.cnt_m[k];
    }
  }
  __syncthreads();
  // ranks
  if (ORDERED && warp < 2 * QN) {
    const bool msg_side = warp < QN;
    const int q = warp % QN;
    const uint32_t side_n = msg_side ? nm : nr, base = msg_side ? nr : 0;
    const int64_t x0 = ((int64_t)side_n * q + QN - 1) / QN, x1 = ((int64_t)side_n * (q + 1) + QN - 1) / QN;
    place_in_order(
        x1 - x0, [&](int64_t x) { return (uint32_t)sm.key[base + x0 + x]; }, sm.start_m, sm.pcnt[warp],
        [&](int64_t x, uint32_t k, uint32_t r, uint32_t slot) {
          const uint32_t e = base + (uint32_t)(x0 + x);
          sm.rank[e] = (uint16_t)r;
          if (msg_side) sm.by_key[slot] = (uint16_t)e;
        },
        lane, lt, K);
  } else if (!ORDERED) {
    for (uint32_t e = tid; e < n; e += NT) {
      const uint16_t k = sm.key[e];
      if (k == kNone) continue;
      const bool is_msg = e >= nr;
      const uint32_t r = fetch_inc16(&sm.pcnt[is_msg ? 0 : RROW][k]);
      sm.rank[e] = (uint16_t)r;
      if (is_msg) sm.by_key[sm.start_m[k] + r] = (uint16_t)e;
    }
  }
  __syncthreads();
  // results in bucket order (coalesced): receive at bucket-sorted position
  // r0 + e, message flags at m0 + e - nr; the queue compaction reads the same
  // order, so per-tuple order (all these levels need) is kept
  uint32_t nmatch = 0;
  for (uint32_t e = tid; e < n; e += NT) {
    const uint16_t k = sm.key[e];
    const uint32_t u = sm.idx[e];
    if (e < nr) {
      int64_t mc = MM_NO_MATCH;
      uint8_t f = 0;
      if (k != kNone && sm.rank[e] < sm.cnt_m[k]) {
        const uint32_t j = sm.by_key[sm.start_m[k] + sm.rank[e]];
        mc = a.M.cookie(0, sm.idx[j], mres, mpb);
        f = 1;
        nmatch++;
      }
      a.out_rc[r0 + e] = a.R.cookie(0, u, rres, rpb);
      a.out_mc[r0 + e] = mc;
      a.rflag[r0 + e] = f;
    } else {
      a.mflag[m0 + e - nr] = (k != kNone && sm.rank[e] < sm.cnt_r[k]) ? 1 : 0;
    }
  }
  for (int o = 16; o; o >>= 1) nmatch += __shfl_xor_sync(kFull, nmatch, o);
  if (lane == 0 && nmatch) atomicAdd(a.n_matched, (unsigned long long)nmatch);
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
  SnapRead rs{a.R, 0, 0}, ms{a.M, 0, 0};
  rs.resid = s.rres;
  ms.resid = s.mres;
  rs.pb = 0;  // single endpoint: pending batch starts at 0
  ms.pb = 0;
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
