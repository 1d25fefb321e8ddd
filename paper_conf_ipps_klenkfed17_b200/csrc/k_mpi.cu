// k_mpi.cu -- full MPI semantics (rows A1-A3 of DESIGN.md §1).
//
// Matrix engine: the paper's scan/reduce (§V.A, Algorithms 1-2,
// l.130-173) re-designed for one warp per endpoint on sm_100a:
//  * the endpoint's message headers are staged once in shared memory with
//    16-byte vector loads (A1); availability is a bit per message, 32 per word;
//  * receives are consumed in posting order; for receive i the warp walks the
//    compatibility row block by block (32 messages per block): each lane tests
//    its message with one masked XOR and `ballot` builds the 32-bit vote word
//    (Algorithm 1); `ffs` of vote & avail picks the earliest admissible
//    available message (Algorithm 2's bidder/ffs step) and lane 0 retires the
//    claim from the availability word.  Blocks whose messages are all taken
//    are skipped without comparing (`first` advances past them);
//  * results and the compaction of both queues (A3, §V.A l.149) are written
//    with ballot/popc prefix ranks, in place (write index <= read index).
// Exactness: receives are processed strictly in posting order and each takes
// the lowest-index available admissible message, i.e. the definition of
// DESIGN.md §2.1; ties cannot occur (message indices are distinct).
#include "mm_kernels.h"

namespace mm {

// out_off[e] = first output slot of endpoint e (exclusive scan of the
// snapshot receive counts); one CTA, each thread a contiguous run of
// endpoints, one block scan.  Also zeroes the batch's pair counter.
__global__ void k_out_offsets(Side R, int n_ep, int64_t* out_off, int64_t out_cap, uint32_t* err,
                              unsigned long long* n_matched) {
  __shared__ int64_t sm[1024 / 32 + 1];
  const int per = (n_ep + (int)blockDim.x - 1) / (int)blockDim.x;
  const int e0 = min(n_ep, (int)threadIdx.x * per), e1 = min(n_ep, e0 + per);
  int64_t v = 0;
  for (int e = e0; e < e1; e++) v += (int64_t)R.q_len[e] + R.pend_count(e);
  int64_t tot;
  int64_t run = block_excl_scan(v, sm, &tot);
  for (int e = e0; e < e1; e++) {
    out_off[e] = run;
    run += (int64_t)R.q_len[e] + R.pend_count(e);
  }
  if (threadIdx.x == 0) {
    out_off[n_ep] = tot;
    if (tot > out_cap) atomicOr(err, kErrOutput);
    if (n_matched) *n_matched = 0ull;
  }
}

// Vector-load the endpoint's k-th..(k+1)-th headers when both come from the
// same contiguous source and the address is 16-byte aligned.
__device__ __forceinline__ void stage_headers(const Side& M, int e, int64_t nm, int64_t mres, int64_t mpb,
                                              uint64_t* sm, int lane) {
  // residual part: queue storage, e * cap is a multiple of 2 when cap is even
  const uint64_t* q = M.q_hdr + (int64_t)e * M.cap;
  const uint64_t* p = M.p_hdr ? M.p_hdr + mpb : nullptr;
  if ((((uintptr_t)q) & 15) == 0 && (((uintptr_t)sm) & 15) == 0) {
    int64_t n2 = mres >> 1;
    for (int64_t k = lane; k < n2; k += 32) {
      uint4 v = reinterpret_cast<const uint4*>(q)[k];
      reinterpret_cast<uint4*>(sm)[k] = v;
    }
    if ((mres & 1) && lane == 0) sm[mres - 1] = q[mres - 1];
  } else {
    for (int64_t k = lane; k < mres; k += 32) sm[k] = q[k];
  }
  int64_t np = nm - mres;
  if (np > 0) {
    uint64_t* d = sm + mres;
    if ((((uintptr_t)p) & 15) == 0 && (((uintptr_t)d) & 15) == 0) {
      int64_t n2 = np >> 1;
      for (int64_t k = lane; k < n2; k += 32) reinterpret_cast<uint4*>(d)[k] = reinterpret_cast<const uint4*>(p)[k];
      if ((np & 1) && lane == 0) d[np - 1] = p[np - 1];
    } else {
      for (int64_t k = lane; k < np; k += 32) d[k] = p[k];
    }
  }
}

__global__ void k_mpi_matrix(MpiArgs a) {
  extern __shared__ __align__(16) uint64_t smem[];
  const int lane = threadIdx.x & 31;
  const int wpb = blockDim.x >> 5;
  const int w = threadIdx.x >> 5;
  const int e = a.ep0 + blockIdx.x * wpb + w;
  if (e >= a.n_ep) return;  // warp-uniform; no block-wide barriers below

  uint64_t* sm_m = smem + (size_t)w * a.warp_smem_words;
  uint32_t* avail = reinterpret_cast<uint32_t*>(sm_m + a.msg_slots);

  const int64_t rres = a.R.q_len[e], mres = a.M.q_len[e];
  const int64_t rpb = a.R.pend_begin(e), mpb = a.M.pend_begin(e);
  const int64_t nr = rres + a.R.pend_count(e), nm = mres + a.M.pend_count(e);
  const int64_t obase = a.out_off[e];
  if (nr > a.R.cap || nm > a.M.cap || nm > a.msg_slots || obase + nr > a.out_cap) {
    // rejected (mm.h): receives reported unmatched if the output holds them,
    // queues left as they were
    if (lane == 0) atomicOr(a.err, kErrCapacity);
    if (obase + nr <= a.out_cap)
      for (int64_t i = lane; i < nr; i += 32) {
        a.out_rc[obase + i] = a.R.cookie(e, i, rres, rpb);
        a.out_mc[obase + i] = (int64_t)MM_NO_MATCH;
      }
    return;
  }

  stage_headers(a.M, e, nm, mres, mpb, sm_m, lane);
  const int nblk = (int)((nm + 31) >> 5);
  for (int b = lane; b < nblk; b += 32) {
    int64_t rem = nm - 32 * (int64_t)b;
    avail[b] = rem >= 32 ? kFull : ((1u << rem) - 1u);
  }
  __syncwarp();

  int first = 0;
  int64_t wr = 0;
  uint32_t matched = 0;
  uint64_t* qrh = a.q_rh_w + (int64_t)e * a.R.cap;
  int64_t* qrc = a.q_rc_w + (int64_t)e * a.R.cap;
  const uint32_t lt = lanemask_lt();

  for (int64_t base = 0; base < nr; base += 32) {
    const int64_t k = base + lane;
    const bool valid = k < nr;
    uint64_t rh = 0;
    int64_t rc = 0;
    if (valid) {
      rh = a.R.hdr(e, k, rres, rpb);
      rc = a.R.cookie(e, k, rres, rpb);
    }
    const uint64_t rmask = wildcard_mask(rh);
    int res = -1;
    const int cnt = (int)min((int64_t)32, nr - base);
    for (int t = 0; t < cnt; t++) {
      const uint64_t r = __shfl_sync(kFull, rh, t);
      const uint64_t msk = __shfl_sync(kFull, rmask, t);
      for (int b = first; b < nblk; b++) {
        const uint32_t av = avail[b];
        if (av == 0) continue;
        const uint64_t m = sm_m[32 * b + lane];
        const uint32_t hit = __ballot_sync(kFull, ((m ^ r) & msk) == 0) & av;
        if (hit) {
          const int bit = __ffs(hit) - 1;
          if (lane == 0) avail[b] = av & ~(1u << bit);
          if (lane == t) res = 32 * b + bit;
          break;
        }
      }
      __syncwarp();
      while (first < nblk && avail[first] == 0) first++;
    }
    if (valid) {
      a.out_rc[obase + k] = rc;
      a.out_mc[obase + k] = res >= 0 ? a.M.cookie(e, res, mres, mpb) : (int64_t)MM_NO_MATCH;
    }
    const uint32_t um = __ballot_sync(kFull, valid && res < 0);
    matched += __popc(__ballot_sync(kFull, valid && res >= 0));
    __syncwarp();  // every lane has read its queue slot before in-place writes
    if (valid && res < 0) {
      const int64_t pos = wr + __popc(um & lt);
      qrh[pos] = rh;
      qrc[pos] = rc;
    }
    wr += __popc(um);
  }

  // compact the unexpected-message queue: survivors keep arrival order
  uint64_t* qmh = a.q_mh_w + (int64_t)e * a.M.cap;
  int64_t* qmc = a.q_mc_w + (int64_t)e * a.M.cap;
  int64_t wm = 0;
  for (int b = 0; b < nblk; b++) {
    const uint32_t av = avail[b];
    const int64_t j = 32 * (int64_t)b + lane;
    const bool keep = (av >> lane) & 1u;
    uint64_t h = 0;
    int64_t c = 0;
    if (keep) {
      h = sm_m[j];
      c = a.M.cookie(e, j, mres, mpb);
    }
    __syncwarp();
    if (keep) {
      const int64_t pos = wm + __popc(av & lt);
      qmh[pos] = h;
      qmc[pos] = c;
    }
    wm += __popc(av);
  }
  if (lane == 0) {
    a.rres_w[e] = (int32_t)wr;
    a.mres_w[e] = (int32_t)wm;
    if (matched) atomicAdd(a.n_matched, (unsigned long long)matched);
  }
}

cudaError_t launch_mpi_matrix(const MpiArgs& a, cudaStream_t st) {
  if (a.n_ep <= a.ep0) return cudaSuccess;
  const size_t per_warp = (size_t)a.warp_smem_words * 8;
  int wpb = (int)(96 * 1024 / per_warp);
  if (wpb > 8) wpb = 8;
  if (wpb < 1) wpb = 1;
  const size_t smem = per_warp * wpb;
  cudaError_t err = ensure_dyn_smem<k_mpi_matrix>(smem);
  if (err != cudaSuccess) return err;
  const int grid = (a.n_ep - a.ep0 + wpb - 1) / wpb;
  count_launch();
  k_mpi_matrix<<<grid, wpb * 32, smem, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_out_offsets(const Side& R, int n_ep, int64_t* out_off, int64_t out_cap, uint32_t* err,
                               unsigned long long* n_matched, cudaStream_t st) {
  count_launch();
  k_out_offsets<<<1, 1024, 0, st>>>(R, n_ep, out_off, out_cap, err, n_matched);
  return cudaGetLastError();
}

}  // namespace mm
