// k_mpi_fifo.cu -- full MPI semantics, key-FIFO engine (rows A2-A3).
//
// Observation: under "each receive, in posting order, takes
// the earliest-arrived unmatched message it admits", every receive consumes
// the HEAD of one per-tuple FIFO -- an exact receive the head of its own
// tuple's list, a wildcard receive the earliest head among the tuples it
// admits.  So the state of an endpoint is one consumption counter per tuple,
// and an exact receive of tuple k at posting position i takes
//     list_k[ e_k(i) + c_k(i) ]   (if < n_k, else nothing),
// with e_k(i) the exact receives of k before i (a prefix count) and c_k(i)
// the wildcard receives before i that took from k (the claims earlier
// wildcards retired from the list).  Only wildcard receives need a search.
//
// Per endpoint (one CTA, workspace in shared memory, or in an L2-resident
// global slice for deep queues):
//  1. stage message headers (16-byte vector loads) and insert them into an
//     open-addressing hash table (16-bit CAS); dense tuple ids by block scan;
//     per-tuple counts and starts by block scan; one warp places messages into
//     their tuple lists in arrival order (match_any ranks), while the other
//     warps classify receives (exact tuple id / wildcard / absent tuple);
//  2. one warp sweeps the receives in posting order, 32 at a time: exact
//     receives between two wildcards resolve together (match_any gives the
//     rank among equal tuples, the per-tuple counters give the prefix); a
//     wildcard receive makes the warp scan the tuples, test admissibility with
//     one masked XOR, read each admitted tuple's head and take the minimum
//     arrival index (redux.sync.min), retiring the claim by bumping c_k;
//  3. results, and the in-place compaction of both queues, are written with
//     ballot/popc prefix ranks.
// Results equal the definition exactly (no ties: arrival indices are unique).
#include "mm_kernels.h"

namespace mm {

constexpr uint32_t kRecvWild = 0xFFFFFFFEu;
constexpr uint32_t kRecvNone = 0xFFFFFFFFu;
constexpr uint16_t kSlotEmpty = 0xFFFFu;

struct FifoWs {
  uint64_t* msgs;      // [mcap] message headers
  uint16_t* table;     // [H] slot -> representative message (kSlotEmpty)
  uint16_t* slot_id;   // [H] slot -> dense tuple id
  uint16_t* key_owner; // [mcap] tuple id -> representative message
  uint32_t* key_cnt;   // [mcap] n_k
  uint32_t* key_start; // [mcap] start of tuple k's list in by_key
  uint32_t* key_e;     // [mcap] exact receives of k seen by the sweep
  uint32_t* key_c;     // [mcap] wildcard receives that took from k
  uint32_t* msg_key;   // [mcap] message -> slot, then -> tuple id
  uint16_t* by_key;    // [mcap] message indices grouped by tuple, arrival order
  uint32_t* recv_key;  // [rcap] receive -> tuple id | kRecvWild | kRecvNone
  uint32_t* matched;   // [mcap/32] message matched bits
};

__device__ __forceinline__ FifoWs carve(uint8_t* base, const FifoLayout& L) {
  FifoWs w;
  w.msgs = reinterpret_cast<uint64_t*>(base + L.msgs);
  w.table = reinterpret_cast<uint16_t*>(base + L.table);
  w.slot_id = reinterpret_cast<uint16_t*>(base + L.slot_id);
  w.key_owner = reinterpret_cast<uint16_t*>(base + L.key_owner);
  w.key_cnt = reinterpret_cast<uint32_t*>(base + L.key_cnt);
  w.key_start = reinterpret_cast<uint32_t*>(base + L.key_start);
  w.key_e = reinterpret_cast<uint32_t*>(base + L.key_e);
  w.key_c = reinterpret_cast<uint32_t*>(base + L.key_c);
  w.msg_key = reinterpret_cast<uint32_t*>(base + L.msg_key);
  w.by_key = reinterpret_cast<uint16_t*>(base + L.by_key);
  w.recv_key = reinterpret_cast<uint32_t*>(base + L.recv_key);
  w.matched = reinterpret_cast<uint32_t*>(base + L.matched);
  return w;
}

// 16-bit CAS on shared or global memory through the containing 32-bit word.
__device__ __forceinline__ uint16_t cas16(uint16_t* p, uint16_t expect, uint16_t val) {
  uint32_t* w = reinterpret_cast<uint32_t*>(reinterpret_cast<uintptr_t>(p) & ~uintptr_t(3));
  const uint32_t sh = (reinterpret_cast<uintptr_t>(p) & 2) ? 16u : 0u;
  uint32_t old = *reinterpret_cast<volatile uint32_t*>(w);
  while (true) {
    const uint16_t cur = (uint16_t)(old >> sh);
    if (cur != expect) return cur;
    const uint32_t nw = (old & ~(0xFFFFu << sh)) | ((uint32_t)val << sh);
    const uint32_t got = atomicCAS(w, old, nw);
    if (got == old) return expect;
    old = got;
  }
}

// Block-wide exclusive scan of per-thread chunk counts (all threads call).
template <int NT>
__device__ __forceinline__ uint32_t block_scan_u32(uint32_t v, uint32_t* sm, uint32_t* total) {
  return block_excl_scan<uint32_t>(v, sm, total);
}

template <int NT>
__global__ void __launch_bounds__(NT) k_mpi_fifo(MpiArgs a, FifoLayout L, uint8_t* gws) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  __shared__ uint32_t scan_sm[NT / 32 + 1];
  __shared__ uint32_t sh_K;
  uint8_t* base = L.in_smem ? smem_raw : gws + (size_t)blockIdx.x * L.total;
  FifoWs ws = carve(base, L);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t lt = lanemask_lt();
  const uint32_t H = L.H, hmask = L.H - 1;

  for (int e = blockIdx.x; e < a.n_ep; e += gridDim.x) {
    const int64_t rres = a.R.q_len[e], mres = a.M.q_len[e];
    const int64_t rpb = a.R.pend_begin(e), mpb = a.M.pend_begin(e);
    const int64_t nr = rres + a.R.pend_count(e), nm = mres + a.M.pend_count(e);
    const int64_t obase = a.out_off[e];
    if (nr > a.R.cap || nm > a.M.cap || obase + nr > a.out_cap) {
      if (tid == 0) atomicOr(a.err, kErrCapacity);
      continue;  // uniform across the CTA
    }

    // ---- 1. stage messages, clear the table -------------------------------
    {
      const uint64_t* q = a.M.q_hdr + (int64_t)e * a.M.cap;
      for (int64_t k = tid; k < mres; k += NT) ws.msgs[k] = q[k];
      const int64_t np = nm - mres;
      const uint64_t* p = a.M.p_hdr ? a.M.p_hdr + mpb : nullptr;
      uint64_t* d = ws.msgs + mres;
      if (np > 0 && ((((uintptr_t)p) | ((uintptr_t)d)) & 15) == 0) {
        for (int64_t k = tid; k < (np >> 1); k += NT)
          reinterpret_cast<uint4*>(d)[k] = reinterpret_cast<const uint4*>(p)[k];
        if ((np & 1) && tid == 0) d[np - 1] = p[np - 1];
      } else {
        for (int64_t k = tid; k < np; k += NT) d[k] = p[k];
      }
      for (uint32_t s = tid; s < H / 2; s += NT) reinterpret_cast<uint32_t*>(ws.table)[s] = 0xFFFFFFFFu;
      for (int64_t k = tid; k < (nm + 31) / 32; k += NT) ws.matched[k] = 0u;
    }
    __syncthreads();
    // insert every message's tuple (linear probing, lock-free)
    for (int64_t j = tid; j < nm; j += NT) {
      const uint64_t h = ws.msgs[j];
      uint32_t s = header_hash(h) & hmask;
      while (true) {
        uint16_t o = ws.table[s];
        if (o == kSlotEmpty) {
          o = cas16(&ws.table[s], kSlotEmpty, (uint16_t)j);
          if (o == kSlotEmpty) break;
        }
        if (ws.msgs[o] == h) break;
        s = (s + 1) & hmask;
      }
      ws.msg_key[j] = s;
    }
    __syncthreads();
    // dense tuple ids in slot order
    {
      const uint32_t per = (H + NT - 1) / NT;
      const uint32_t s0 = tid * per, s1 = min(H, s0 + per);
      uint32_t c = 0;
      for (uint32_t s = s0; s < s1; s++) c += ws.table[s] != kSlotEmpty;
      uint32_t tot;
      uint32_t id = block_scan_u32<NT>(c, scan_sm, &tot);
      for (uint32_t s = s0; s < s1; s++) {
        const uint16_t o = ws.table[s];
        if (o != kSlotEmpty) {
          ws.slot_id[s] = (uint16_t)id;
          ws.key_owner[id] = o;
          ws.key_cnt[id] = 0;
          ws.key_e[id] = 0;
          ws.key_c[id] = 0;
          id++;
        }
      }
      if (tid == 0) sh_K = tot;
    }
    __syncthreads();
    const uint32_t K = sh_K;
    for (int64_t j = tid; j < nm; j += NT) {
      const uint32_t id = ws.slot_id[ws.msg_key[j]];
      ws.msg_key[j] = id;
      atomicAdd(&ws.key_cnt[id], 1u);
    }
    __syncthreads();
    {
      const uint32_t per = (K + NT - 1) / NT;
      const uint32_t k0 = min(K, tid * per), k1 = min(K, k0 + per);
      uint32_t c = 0;
      for (uint32_t k = k0; k < k1; k++) c += ws.key_cnt[k];
      uint32_t tot;
      uint32_t st = block_scan_u32<NT>(c, scan_sm, &tot);
      for (uint32_t k = k0; k < k1; k++) {
        ws.key_start[k] = st;
        st += ws.key_cnt[k];
      }
    }
    __syncthreads();
    if (warp == 0) {
      // place messages into their tuple lists in arrival order (key_e is the
      // running count here and is cleared again below)
      for (int64_t b = 0; b < nm; b += 32) {
        const int64_t j = b + lane;
        const uint32_t id = j < nm ? ws.msg_key[j] : 0xFFFFFFFFu;
        const uint32_t peers = __match_any_sync(kFull, id);
        if (j < nm) {
          const uint32_t run = ws.key_e[id];
          ws.by_key[ws.key_start[id] + run + __popc(peers & lt)] = (uint16_t)j;
          __syncwarp(peers);
          if ((peers >> lane) == 1u) ws.key_e[id] = run + __popc(peers);
        }
        __syncwarp();
      }
    } else {
      // classify receives: exact tuple id, wildcard, or a tuple no message has
      for (int64_t i = tid - 32; i < nr; i += NT - 32) {
        const uint64_t h = a.R.hdr(e, i, rres, rpb);
        uint32_t rk;
        if (wildcard_mask(h) != ~0ull) {
          rk = kRecvWild;
        } else {
          rk = kRecvNone;
          uint32_t s = header_hash(h) & hmask;
          while (true) {
            const uint16_t o = ws.table[s];
            if (o == kSlotEmpty) break;
            if (ws.msgs[o] == h) {
              rk = ws.slot_id[s];
              break;
            }
            s = (s + 1) & hmask;
          }
        }
        ws.recv_key[i] = rk;
      }
    }
    __syncthreads();
    for (uint32_t k = tid; k < K; k += NT) ws.key_e[k] = 0;
    __syncthreads();

    // ---- 2. in-order sweep (one warp) --------------------------------------
    if (warp == 0) {
      uint64_t* qrh = a.q_rh_w + (int64_t)e * a.R.cap;
      int64_t* qrc = a.q_rc_w + (int64_t)e * a.R.cap;
      int64_t wr = 0;
      uint32_t nmatch = 0;
      // software pipeline: the next chunk's headers/cookies are in flight
      // while the current chunk resolves
      uint64_t nrh = 0;
      int64_t nrc = 0;
      if (lane < nr) {
        nrh = a.R.hdr(e, lane, rres, rpb);
        nrc = a.R.cookie(e, lane, rres, rpb);
      }
      for (int64_t b0 = 0; b0 < nr; b0 += 32) {
        const int64_t i = b0 + lane;
        const bool valid = i < nr;
        const uint64_t rh = nrh;
        const int64_t rc = nrc;
        if (i + 32 < nr) {
          nrh = a.R.hdr(e, i + 32, rres, rpb);
          nrc = a.R.cookie(e, i + 32, rres, rpb);
        }
        const uint32_t rk = valid ? ws.recv_key[i] : kRecvNone;
        int64_t res = -1;
        uint32_t wmask = __ballot_sync(kFull, valid && rk == kRecvWild);
        int seg = 0;
        while (true) {
          const int t = wmask ? __ffs(wmask) - 1 : 32;
          // exact receives in lanes [seg, t)
          const bool in = valid && lane >= seg && lane < t && rk < kRecvWild;
          const uint32_t key = in ? rk : 0xFFFFFFFFu;
          const uint32_t peers = __match_any_sync(kFull, key);
          uint32_t e0 = 0;
          if (in) {
            e0 = ws.key_e[rk];
            const uint32_t hd = e0 + __popc(peers & lt) + ws.key_c[rk];
            if (hd < ws.key_cnt[rk]) {
              const uint32_t j = ws.by_key[ws.key_start[rk] + hd];
              res = j;
              atomicOr(&ws.matched[j >> 5], 1u << (j & 31));
            }
          }
          __syncwarp();
          if (in && (peers >> lane) == 1u) ws.key_e[rk] = e0 + __popc(peers);
          __syncwarp();
          if (t == 32) break;
          // wildcard receive at lane t: earliest head among admitted tuples
          const uint64_t r = __shfl_sync(kFull, rh, t);
          const uint64_t msk = wildcard_mask(r);
          uint32_t best = 0xFFFFFFFFu, bestk = 0;
          for (uint32_t k = lane; k < K; k += 32) {
            if (((ws.msgs[ws.key_owner[k]] ^ r) & msk) == 0) {
              const uint32_t hd = ws.key_e[k] + ws.key_c[k];
              if (hd < ws.key_cnt[k]) {
                const uint32_t j = ws.by_key[ws.key_start[k] + hd];
                if (j < best) {
                  best = j;
                  bestk = k;
                }
              }
            }
          }
          const uint32_t win = __reduce_min_sync(kFull, best);
          if (win != 0xFFFFFFFFu) {
            if (best == win) {
              ws.key_c[bestk] += 1;
              atomicOr(&ws.matched[win >> 5], 1u << (win & 31));
            }
            if (lane == t) res = win;
          }
          __syncwarp();
          wmask &= ~(1u << t);
          seg = t + 1;
        }
        if (valid) {
          a.out_rc[obase + i] = rc;
          a.out_mc[obase + i] = res >= 0 ? a.M.cookie(e, res, mres, mpb) : (int64_t)MM_NO_MATCH;
        }
        const uint32_t um = __ballot_sync(kFull, valid && res < 0);
        nmatch += __popc(__ballot_sync(kFull, valid && res >= 0));
        __syncwarp();
        if (valid && res < 0) {
          const int64_t pos = wr + __popc(um & lt);
          qrh[pos] = rh;
          qrc[pos] = rc;
        }
        wr += __popc(um);
      }
      if (lane == 0) {
        a.rres_w[e] = (int32_t)wr;
        if (nmatch) atomicAdd(a.n_matched, (unsigned long long)nmatch);
      }
    }
    __syncthreads();
    // ---- 3. compact the unexpected-message queue (warp 1, or 0) -----------
    if (warp == (NT > 32 ? 1 : 0)) {
      uint64_t* qmh = a.q_mh_w + (int64_t)e * a.M.cap;
      int64_t* qmc = a.q_mc_w + (int64_t)e * a.M.cap;
      int64_t wm = 0;
      for (int64_t b0 = 0; b0 < nm; b0 += 32) {
        const int64_t j = b0 + lane;
        const bool keep = j < nm && !((ws.matched[j >> 5] >> (j & 31)) & 1u);
        uint64_t h = 0;
        int64_t c = 0;
        if (keep) {
          h = ws.msgs[j];
          c = a.M.cookie(e, j, mres, mpb);
        }
        const uint32_t km = __ballot_sync(kFull, keep);
        __syncwarp();
        if (keep) {
          const int64_t pos = wm + __popc(km & lt);
          qmh[pos] = h;
          qmc[pos] = c;
        }
        wm += __popc(km);
      }
      if (lane == 0) a.mres_w[e] = (int32_t)wm;
    }
    __syncthreads();  // the workspace is reused by the next endpoint
  }
}

FifoLayout fifo_layout(int64_t rcap, int64_t mcap) {
  FifoLayout L;
  int64_t H = 1;
  while (H < 2 * mcap) H <<= 1;
  if (H < 64) H = 64;
  L.H = (uint32_t)H;
  int64_t off = 0;
  auto take = [&](int64_t bytes) {
    int64_t o = off;
    off += (bytes + 15) / 16 * 16;
    return o;
  };
  L.msgs = take(8 * mcap);
  L.table = take(2 * H);
  L.slot_id = take(2 * H);
  L.key_owner = take(2 * mcap);
  L.key_cnt = take(4 * mcap);
  L.key_start = take(4 * mcap);
  L.key_e = take(4 * mcap);
  L.key_c = take(4 * mcap);
  L.msg_key = take(4 * mcap);
  L.by_key = take(2 * mcap);
  L.recv_key = take(4 * rcap);
  L.matched = take(4 * ((mcap + 31) / 32));
  L.total = off;
  L.in_smem = off <= kFifoSmemMax;
  return L;
}

int fifo_grid(const FifoLayout& L, int n_ep) {
  if (L.in_smem) return n_ep;
  int g = 148 * 2;
  return n_ep < g ? n_ep : g;
}

cudaError_t launch_mpi_fifo(const MpiArgs& a, const FifoLayout& L, uint8_t* gws, cudaStream_t st) {
  if (a.n_ep <= 0) return cudaSuccess;
  const int grid = fifo_grid(L, a.n_ep);
  cudaError_t err;
  if (L.in_smem) {
    err = cudaFuncSetAttribute(k_mpi_fifo<128>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)L.total);
    if (err != cudaSuccess) return err;
    count_launch();
    k_mpi_fifo<128><<<grid, 128, (size_t)L.total, st>>>(a, L, nullptr);
  } else {
    count_launch();
    k_mpi_fifo<512><<<grid, 512, 0, st>>>(a, L, gws);
  }
  return cudaGetLastError();
}

}  // namespace mm
