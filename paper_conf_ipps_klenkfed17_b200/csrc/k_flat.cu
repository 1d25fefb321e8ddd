// k_flat.cu -- the no-wildcard levels (rows A4, A5), queue compaction (A3)
// for them, pending-batch materialisation and mm_route's partition (A6).
//
// Ordered level (§VI.A, Table II rows 3-4): with wildcards
// prohibited the per-tuple FIFO makes the MPI result a rank pairing -- the
// n-th posted receive of a tuple takes the n-th arrived message of it.  It is
// computed by a stable LSD radix sort of [receives ++ messages] over only the
// header bits that vary in the batch, then one scan that finds each run of
// equal tuples (receives precede messages in a run because the sort is
// stable) and a pairing pass.
//
// Unordered level (§VI.C, Table II rows 5-6): a lock-free
// open-addressing hash table in HBM.  Receives insert their tuple (32-bit CAS
// on the slot owner, linear probing) and draw a ticket from the slot's
// receive counter; the ticket (slot, t) is filed in a second table.  Each
// message finds its tuple's slot, draws a ticket from the message counter and,
// if a receive holds that ticket, takes it.  Per tuple exactly
// min(#recv, #msg) pairs form; which receive gets which message is the
// nondeterminism the relaxation allows.
#include "mm_kernels.h"

namespace mm {

// ------------------------------------------------------------ snapshot info
__global__ void k_snapshot_info(Side R, Side M, int64_t bound, SnapInfo* info, bool want_diff) {
  const int64_t rres = R.q_len[0], mres = M.q_len[0];
  const int64_t nr = rres + R.pend_count(0), nm = mres + M.pend_count(0);
  const int64_t rpb = R.pend_begin(0), mpb = M.pend_begin(0);
  uint64_t ref = nr > 0 ? R.hdr(0, 0, rres, rpb) : (nm > 0 ? M.hdr(0, 0, mres, mpb) : 0ull);
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    info->ref = ref;
    info->rres = (int32_t)rres;
    info->mres = (int32_t)mres;
  }
  if (!want_diff) return;
  const int64_t n = nr + nm;
  uint64_t d = 0;
  for (int64_t u = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; u < n && u < bound;
       u += (int64_t)gridDim.x * blockDim.x) {
    uint64_t h = u < nr ? R.hdr(0, u, rres, rpb) : M.hdr(0, u - nr, mres, mpb);
    d |= h ^ ref;
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) d |= __shfl_xor_sync(kFull, d, o);
  if ((threadIdx.x & 31) == 0 && d) atomicOr(&info->diff, (unsigned long long)d);
}

cudaError_t launch_snapshot_info(const Side& R, const Side& M, int64_t bound, SnapInfo* info, bool want_diff,
                                 cudaStream_t st) {
  cudaError_t err = cudaMemsetAsync(info, 0, sizeof(SnapInfo), st);
  if (err != cudaSuccess) return err;
  int64_t blocks = want_diff ? (bound + 255) / 256 : 1;
  if (blocks > 148 * 16) blocks = 148 * 16;
  if (blocks < 1) blocks = 1;
  count_launch();
  k_snapshot_info<<<(unsigned)blocks, 256, 0, st>>>(R, M, bound, info, want_diff);
  return cudaGetLastError();
}

// -------------------------------------------------------- sort-and-rank (A4)
// Gather plan: the varying bits of the batch as runs (shift, len) of the
// header word, packed into the low bits of the sort key.
struct BitPlan {
  int n;
  uint8_t shift[64];
  uint8_t len[64];
};

__device__ __forceinline__ uint64_t gather_bits(uint64_t x, const BitPlan& p) {
  uint64_t out = 0;
  int pos = 0;
  for (int i = 0; i < p.n; i++) {
    const int l = p.len[i];
    const uint64_t m = l >= 64 ? ~0ull : ((1ull << l) - 1ull);
    out |= ((x >> p.shift[i]) & m) << pos;
    pos += l;
  }
  return out;
}

__global__ void k_sort_prep(FlatArgs a, uint64_t ref, BitPlan plan, uint64_t* key, uint32_t* val) {
  const int64_t n = a.nr + a.nm;
  const int64_t rres = a.R.q_len[0], mres = a.M.q_len[0];
  const int64_t rpb = a.R.pend_begin(0), mpb = a.M.pend_begin(0);
  for (int64_t u = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; u < n; u += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t h = u < a.nr ? a.R.hdr(0, u, rres, rpb) : a.M.hdr(0, u - a.nr, mres, mpb);
    key[u] = gather_bits(h ^ ref, plan);
    val[u] = (uint32_t)u;
  }
}

struct DigitOf {
  const uint64_t* key;
  int shift;
  __device__ __forceinline__ uint32_t operator()(int64_t k) const { return (uint32_t)(key[k] >> shift) & 255u; }
  __device__ __forceinline__ uint32_t of_payload(int64_t, uint64_t a, uint64_t) const {
    return (uint32_t)(a >> shift) & 255u;
  }
};
struct MoveKV {
  const uint64_t* ki;
  const uint32_t* vi;
  uint64_t* ko;
  uint32_t* vo;
  __device__ __forceinline__ void load(int64_t k, uint64_t& a, uint64_t& b) const {
    a = ki[k];
    b = vi[k];
  }
  __device__ __forceinline__ void store(int64_t dst, uint64_t a, uint64_t b) const {
    ko[dst] = a;
    vo[dst] = (uint32_t)b;
  }
};

// Run boundaries: value(p) = (head << 32) | is_receive, scanned.
struct RunIn {
  const uint64_t* key;
  const uint32_t* val;
  int64_t nr;
  __device__ __forceinline__ unsigned long long operator()(int64_t p) const {
    const unsigned long long h = (p == 0 || key[p] != key[p - 1]) ? 1ull : 0ull;
    return (h << 32) | (val[p] < (uint64_t)nr ? 1ull : 0ull);
  }
};
struct RunOut {
  uint32_t* rid;
  uint32_t* run_start;
  uint32_t* run_rc;
  int64_t n;
  __device__ __forceinline__ void operator()(int64_t p, unsigned long long ex, unsigned long long v) const {
    const uint32_t h = (uint32_t)(v >> 32), isr = (uint32_t)v;
    const uint32_t r = (uint32_t)(ex >> 32) + h - 1u;
    const uint32_t crx = (uint32_t)ex;
    rid[p] = r;
    if (h) {
      run_start[r] = (uint32_t)p;
      run_rc[r] = crx;
    }
    if (p == n - 1) {
      run_start[r + 1] = (uint32_t)n;
      run_rc[r + 1] = crx + isr;
    }
  }
};

__global__ void k_pair(FlatArgs a, const uint32_t* val, const uint32_t* rid, const uint32_t* run_start,
                       const uint32_t* run_rc) {
  unsigned long long* n_matched = a.n_matched;
  const int64_t n = a.nr + a.nm;
  const int64_t rres = a.R.q_len[0], mres = a.M.q_len[0];
  const int64_t rpb = a.R.pend_begin(0), mpb = a.M.pend_begin(0);
  uint32_t cnt = 0;
  for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < n; p += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t r = rid[p];
    const int64_t s = run_start[r], e = run_start[r + 1];
    const int64_t nR = (int64_t)run_rc[r + 1] - run_rc[r];
    const int64_t u = val[p];
    if (u < a.nr) {
      const int64_t q = s + nR + (p - s);  // partner position: same rank among the run's messages
      const bool m = q < e;
      a.out_rc[u] = a.R.cookie(0, u, rres, rpb);
      a.out_mc[u] = m ? a.M.cookie(0, (int64_t)val[q] - a.nr, mres, mpb) : (int64_t)MM_NO_MATCH;
      a.rflag[u] = m;
      cnt += m;
    } else {
      a.mflag[u - a.nr] = (p - s - nR) < nR;
    }
  }
  for (int o = 16; o; o >>= 1) cnt += __shfl_xor_sync(kFull, cnt, o);
  if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(n_matched, (unsigned long long)cnt);
}

static int grid_for(int64_t n, int threads) {
  int64_t b = (n + threads - 1) / threads;
  if (b > 148 * 32) b = 148 * 32;
  return b < 1 ? 1 : (int)b;
}

cudaError_t run_sort_rank(const FlatArgs& a, uint64_t ref, uint64_t diff, const SortScratch& s, cudaStream_t st) {
  const int64_t n = a.nr + a.nm;
  if (n == 0) return cudaSuccess;
  BitPlan plan{};
  int nbits = 0;
  for (int b = 0; b < 64;) {
    if (!((diff >> b) & 1ull)) {
      b++;
      continue;
    }
    int l = 0;
    while (b + l < 64 && ((diff >> (b + l)) & 1ull)) l++;
    plan.shift[plan.n] = (uint8_t)b;
    plan.len[plan.n] = (uint8_t)l;
    plan.n++;
    nbits += l;
    b += l;
  }
  count_launch();
  k_sort_prep<<<grid_for(n, 256), 256, 0, st>>>(a, ref, plan, s.key[0], s.val[0]);
  cudaError_t err = cudaGetLastError();
  if (err != cudaSuccess) return err;
  int cur = 0;
  for (int sh = 0; sh < nbits; sh += 8) {
    err = partition_stable(DigitOf{s.key[cur], sh}, MoveKV{s.key[cur], s.val[cur], s.key[cur ^ 1], s.val[cur ^ 1]}, n,
                           256, s.part, st);
    if (err != cudaSuccess) return err;
    cur ^= 1;
  }
  err = scan_apply<unsigned long long>(RunIn{s.key[cur], s.val[cur], a.nr}, n, s.scan,
                                       RunOut{s.rid, s.run_start, s.run_rc, n}, st);
  if (err != cudaSuccess) return err;
  count_launch();
  k_pair<<<grid_for(n, 256), 256, 0, st>>>(a, s.val[cur], s.rid, s.run_start, s.run_rc);
  return cudaGetLastError();
}

// -------------------------------------------------------------- hash (A5)
constexpr uint32_t kEmpty = 0xFFFFFFFFu;

__device__ __forceinline__ uint32_t ticket_hash(uint32_t slot, uint32_t t) {
  return jenkins32(slot ^ jenkins32(t ^ 0x9e3779b9u));
}

__global__ void k_hash_insert(FlatArgs a, HashScratch h) {
  const int64_t rres = a.R.q_len[0], rpb = a.R.pend_begin(0);
  const uint32_t mask = (uint32_t)(h.T - 1);
  for (int64_t u = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; u < a.nr; u += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t key = a.R.hdr(0, u, rres, rpb);
    uint32_t s = header_hash(key) & mask;
    while (true) {
      uint32_t o = h.owner[s];
      if (o == kEmpty) {
        o = atomicCAS(&h.owner[s], kEmpty, (uint32_t)u);
        if (o == kEmpty) break;  // this receive now represents the tuple
      }
      if (a.R.hdr(0, o, rres, rpb) == key) break;
      s = (s + 1) & mask;
    }
    const uint32_t t = atomicAdd(&h.rcnt[s], 1u);
    const unsigned long long tk = ((unsigned long long)s << 32) | t;
    uint32_t s2 = ticket_hash(s, t) & mask;
    while (atomicCAS(&h.tkey[s2], ~0ull, tk) != ~0ull) s2 = (s2 + 1) & mask;
    h.tval[s2] = (uint32_t)u;
    a.out_rc[u] = a.R.cookie(0, u, rres, rpb);
    a.out_mc[u] = MM_NO_MATCH;
    a.rflag[u] = 0;
  }
}

__global__ void k_hash_probe(FlatArgs a, HashScratch h) {
  unsigned long long* n_matched = a.n_matched;
  const int64_t rres = a.R.q_len[0], rpb = a.R.pend_begin(0);
  const int64_t mres = a.M.q_len[0], mpb = a.M.pend_begin(0);
  const uint32_t mask = (uint32_t)(h.T - 1);
  uint32_t cnt = 0;
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < a.nm; v += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t key = a.M.hdr(0, v, mres, mpb);
    uint32_t s = header_hash(key) & mask;
    bool found = false;
    while (true) {
      const uint32_t o = h.owner[s];
      if (o == kEmpty) break;
      if (a.R.hdr(0, o, rres, rpb) == key) {
        found = true;
        break;
      }
      s = (s + 1) & mask;
    }
    uint8_t got = 0;
    if (found) {
      const uint32_t t = atomicAdd(&h.mcnt[s], 1u);
      if (t < h.rcnt[s]) {
        const unsigned long long tk = ((unsigned long long)s << 32) | t;
        uint32_t s2 = ticket_hash(s, t) & mask;
        while (h.tkey[s2] != tk) s2 = (s2 + 1) & mask;
        const uint32_t u = h.tval[s2];
        a.out_mc[u] = a.M.cookie(0, v, mres, mpb);
        a.rflag[u] = 1;
        got = 1;
      }
    }
    a.mflag[v] = got;
    cnt += got;
  }
  for (int o = 16; o; o >>= 1) cnt += __shfl_xor_sync(kFull, cnt, o);
  if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(n_matched, (unsigned long long)cnt);
}

cudaError_t run_hash(const FlatArgs& a, const HashScratch& h, cudaStream_t st) {
  cudaError_t err;
  if ((err = cudaMemsetAsync(h.owner, 0xFF, (size_t)h.T * 4, st)) != cudaSuccess) return err;
  if ((err = cudaMemsetAsync(h.rcnt, 0, (size_t)h.T * 4, st)) != cudaSuccess) return err;
  if ((err = cudaMemsetAsync(h.mcnt, 0, (size_t)h.T * 4, st)) != cudaSuccess) return err;
  if ((err = cudaMemsetAsync(h.tkey, 0xFF, (size_t)h.T * 8, st)) != cudaSuccess) return err;
  if (a.nr > 0) {
    count_launch();
    k_hash_insert<<<grid_for(a.nr, 256), 256, 0, st>>>(a, h);
  }
  if (a.nm > 0) {
    count_launch();
    k_hash_probe<<<grid_for(a.nm, 256), 256, 0, st>>>(a, h);
  }
  return cudaGetLastError();
}

// ----------------------------------------------------------- compaction (A3)
struct UnmatchedIn {
  const uint8_t* matched;
  __device__ __forceinline__ uint32_t operator()(int64_t u) const { return matched[u] ? 0u : 1u; }
};
struct CompactOut {
  Side S;
  int64_t resid, pb, n;
  uint64_t* q_h;
  int64_t* q_c;
  int32_t* q_len;
  __device__ __forceinline__ void operator()(int64_t u, uint32_t ex, uint32_t v) const {
    if (v) {
      q_h[ex] = S.hdr(0, u, resid, pb);
      q_c[ex] = S.cookie(0, u, resid, pb);
    }
    if (u == n - 1) *q_len = (int32_t)(ex + v);
  }
};

__global__ void k_set_len(int32_t* q_len, int32_t v) { *q_len = v; }

cudaError_t run_compact(const Side& S, int64_t resid, int64_t n, const uint8_t* matched, uint64_t* q_h,
                        int64_t* q_c, int32_t* q_len, uint32_t* scan, cudaStream_t st) {
  if (n == 0) {
    count_launch();
    k_set_len<<<1, 1, 0, st>>>(q_len, 0);
    return cudaGetLastError();
  }
  // S's pend_begin(0) is evaluated on the device side by the functor via pb;
  // for the single-endpoint levels it is p_off ? p_off[0] : 0 == 0.
  return scan_apply<uint32_t>(UnmatchedIn{matched}, n, scan, CompactOut{S, resid, 0, n, q_h, q_c, q_len}, st);
}

// -------------------------------------------------------------- materialise
__global__ void k_materialize(Side S, int n_ep, uint64_t* q_h, int64_t* q_c, const int32_t* q_len, uint32_t* err) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < S.p_n; i += (int64_t)gridDim.x * blockDim.x) {
    int e = 0;
    if (S.p_off) {
      int lo = 0, hi = n_ep;  // largest e with p_off[e] <= i
      while (hi - lo > 1) {
        int mid = (lo + hi) >> 1;
        if (S.p_off[mid] <= i) lo = mid;
        else hi = mid;
      }
      e = lo;
    }
    const int64_t k = i - S.pend_begin(e);
    const int64_t pos = (int64_t)q_len[e] + k;
    if ((int64_t)q_len[e] + S.pend_count(e) <= S.cap) {
      q_h[(int64_t)e * S.cap + pos] = S.p_hdr[i];
      q_c[(int64_t)e * S.cap + pos] = S.p_cookie ? S.p_cookie[i] : S.p_seq0 + i;
    } else if (k == 0) {
      atomicOr(err, kErrCapacity);  // the endpoint's pending batch does not fit: dropped whole (mm.h)
    }
  }
}
__global__ void k_materialize_len(Side S, int n_ep, int32_t* q_len) {
  for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < n_ep; e += gridDim.x * blockDim.x) {
    const int64_t v = (int64_t)q_len[e] + S.pend_count(e);
    if (v <= S.cap) q_len[e] = (int32_t)v;  // else rejected: the queue keeps its contents
  }
}

cudaError_t launch_materialize(const Side& S, int n_ep, uint64_t* q_h, int64_t* q_c, int32_t* q_len, uint32_t* err,
                               cudaStream_t st) {
  if (S.p_n > 0) {
    count_launch();
    k_materialize<<<grid_for(S.p_n, 256), 256, 0, st>>>(S, n_ep, q_h, q_c, q_len, err);
  }
  count_launch();
  k_materialize_len<<<grid_for(n_ep, 256), 256, 0, st>>>(S, n_ep, q_len);
  return cudaGetLastError();
}

// ------------------------------------------------------------------ finalize
// mm_reset: both queues' current lengths and the error flags in one launch
__global__ void k_reset(int32_t* rlen, int32_t* mlen, int n_ep, uint32_t* err, unsigned long long* n_matched) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n_ep; i += gridDim.x * blockDim.x) {
    rlen[i] = 0;
    mlen[i] = 0;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    *err = 0u;
    *n_matched = 0ull;
  }
}
cudaError_t launch_reset(int32_t* rlen, int32_t* mlen, int n_ep, uint32_t* err, unsigned long long* n_matched,
                         cudaStream_t st) {
  count_launch();
  int grid = (n_ep + 255) / 256;
  if (grid > 148 * 4) grid = 148 * 4;
  k_reset<<<grid < 1 ? 1 : grid, 256, 0, st>>>(rlen, mlen, n_ep, err, n_matched);
  return cudaGetLastError();
}

// {n_out, n_matched} into the engine's counts and, if given, the caller's
// device counts (one launch instead of a kernel and a copy)
__global__ void k_finalize(const int64_t* n_out_src, int64_t n_out_host, const unsigned long long* n_matched,
                           int64_t* counts, int64_t* user_counts) {
  const int64_t a = n_out_src ? *n_out_src : n_out_host, b = (int64_t)*n_matched;
  counts[0] = a;
  counts[1] = b;
  if (user_counts) {
    user_counts[0] = a;
    user_counts[1] = b;
  }
}
// Device-decided tail of a bucketed no-wildcard batch (mm_engine.cu,
// FlatTail): the overflow flag and the pair count pick the graph's
// conditional bodies -- the global fallback + compaction, or each side's
// compaction when it is not fully matched -- so the host never reads them
// back; a fully matched side's residual queue is emptied here.
// Without a fallback the pair count is final here, so the gate also writes
// the counts (the fallback body ends with its own finalize).
__global__ void k_flat_gate(const uint32_t* over, const unsigned long long* n_matched, int64_t nr, int64_t nm,
                            cudaGraphConditionalHandle hfb, cudaGraphConditionalHandle hr,
                            cudaGraphConditionalHandle hm, cudaGraphConditionalHandle hany, int32_t* len_r,
                            int32_t* len_m, unsigned long long* fallbacks, int64_t* counts, int64_t* user_counts) {
  const bool fb = *over != 0;
  const unsigned long long m = *n_matched;
  const bool pr = !fb && (int64_t)m != nr, pm = !fb && (int64_t)m != nm;
  cudaGraphSetConditional(hfb, fb ? 1u : 0u);
  cudaGraphSetConditional(hr, pr ? 1u : 0u);
  cudaGraphSetConditional(hm, pm ? 1u : 0u);
  cudaGraphSetConditional(hany, (fb || pr || pm) ? 1u : 0u);
  if (!fb && !pr) *len_r = 0;
  if (!fb && !pm) *len_m = 0;
  if (fb) {
    *fallbacks += 1ull;
  } else {
    counts[0] = nr;
    counts[1] = (int64_t)m;
    if (user_counts) {
      user_counts[0] = nr;
      user_counts[1] = (int64_t)m;
    }
  }
}
cudaError_t launch_flat_gate(const uint32_t* over, const unsigned long long* n_matched, int64_t nr, int64_t nm,
                             cudaGraphConditionalHandle hfb, cudaGraphConditionalHandle hr,
                             cudaGraphConditionalHandle hm, cudaGraphConditionalHandle hany, int32_t* len_r,
                             int32_t* len_m, unsigned long long* fallbacks, int64_t* counts, int64_t* user_counts,
                             cudaStream_t st) {
  count_launch();
  k_flat_gate<<<1, 1, 0, st>>>(over, n_matched, nr, nm, hfb, hr, hm, hany, len_r, len_m, fallbacks, counts,
                               user_counts);
  return cudaGetLastError();
}

cudaError_t launch_finalize(const int64_t* n_out_src, int64_t n_out_host, const unsigned long long* n_matched,
                            int64_t* counts, int64_t* user_counts, cudaStream_t st) {
  count_launch();
  k_finalize<<<1, 1, 0, st>>>(n_out_src, n_out_host, n_matched, counts, user_counts);
  return cudaGetLastError();
}

// --------------------------------------------------------------- route (A6)
struct OwnerOf {
  const uint64_t* a;
  const int64_t* b;
  int world, by;
  // by == 1: bucket = origin rank (bits 40..63 of the cookie a);
  // by == 2: bucket = 2 origin + (b == MM_NO_MATCH) (results split into the
  //          matched and the unmatched receives of each origin).
  // A cookie whose origin bits name no rank goes to the last bucket, placed
  // after every owner's group and left out of the counts.
  __device__ __forceinline__ uint32_t of_payload(int64_t, uint64_t x, uint64_t y) const {
    if (by == 1) {
      const uint64_t o = x >> 40;
      return o < (uint64_t)world ? (uint32_t)o : (uint32_t)world;
    }
    if (by == 2) {
      const uint64_t o = x >> 40;
      return o < (uint64_t)world ? (uint32_t)(2 * o + ((int64_t)y == (int64_t)MM_NO_MATCH)) : (uint32_t)(2 * world);
    }
    return (uint32_t)(((unsigned long long)header_hash(x) * (unsigned)world) >> 32);
  }
  __device__ __forceinline__ uint32_t operator()(int64_t k) const {
    return of_payload(k, a[k], by == 2 ? (uint64_t)b[k] : 0);
  }
};
struct MoveRoute {
  const uint64_t* a;
  const int64_t* b;
  uint64_t* oa;
  int64_t* ob;
  int64_t base;
  __device__ __forceinline__ void load(int64_t k, uint64_t& x, uint64_t& y) const {
    x = a[k];
    y = (uint64_t)(b ? b[k] : (base + k));
  }
  __device__ __forceinline__ void store(int64_t dst, uint64_t x, uint64_t y) const {
    oa[dst] = x;
    ob[dst] = (int64_t)y;
  }
};
__global__ void k_route_counts(const uint32_t* hist, int64_t ntiles, int world, int nb, int64_t n, int64_t* counts) {
  for (int w = threadIdx.x; w < world; w += blockDim.x) {
    int64_t s = hist[(int64_t)w * ntiles];
    int64_t e = w + 1 < nb ? (int64_t)hist[(int64_t)(w + 1) * ntiles] : n;
    counts[w] = e - s;
  }
}

cudaError_t run_route(const uint64_t* a, const int64_t* b, int64_t n, int world, int by, int64_t cookie_base, uint64_t* out_a,
                      int64_t* out_b, int64_t* counts, uint32_t* part, cudaStream_t st) {
  if (n == 0) return cudaMemsetAsync(counts, 0, sizeof(int64_t) * (by == 2 ? 2 * world : world), st);
  const int nc = by == 2 ? 2 * world : world;  // counted buckets
  const int nb = by == 0 ? world : nc + 1;      // + the bucket of cookies naming no rank
  cudaError_t err =
      partition_stable(OwnerOf{a, b, world, by}, MoveRoute{a, b, out_a, out_b, cookie_base}, n, nb, part, st);
  if (err != cudaSuccess) return err;
  int64_t nt = (n + kPartTile - 1) / kPartTile;
  count_launch();
  k_route_counts<<<1, 256, 0, st>>>(part, nt, nc, nb, n, counts);
  return cudaGetLastError();
}

}  // namespace mm
