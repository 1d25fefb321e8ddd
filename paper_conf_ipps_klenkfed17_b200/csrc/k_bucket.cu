// k_bucket.cu -- the no-wildcard levels as hash-bucketed rank pairing
// (rows A4, A5 of DESIGN.md §1; §7.3).
//
// Without wildcards a receive can only take a message with the identical
// tuple, so the tuple key space partitions (§VI.A l.196; §VI.C
// l.215).  Both levels therefore
//  1. partition receives and messages by a hash of the tuple into B buckets
//     (~512 elements per side on average) with MSD passes of <= 10 bits
//     (k_part_pass) into fixed-capacity regions: coalesced runs, one global
//     reservation per digit and tile, no histogram passes; the snapshot
//     index travels with the header;
//  2. match every bucket in one CTA, entirely in shared memory
//     (k_bucket_match): tuples get dense ids, elements are grouped by tuple,
//     NOWILD_ORDERED re-orders each group by snapshot index, and the receive
//     at group position j takes the message at position j -- the n-th receive
//     of a tuple takes the n-th message (the MPI result without wildcards);
//     NOWILD_UNORDERED pairs in whatever order the groups formed (a maximal
//     pairing of equal tuples, what the relaxation allows);
//  3. write results at the bucket's output offset and a matched byte per slot
//     for the queue compaction.
// A bucket larger than its region or than the on-chip capacity raises a flag;
// the host then runs the global sort-and-rank (ordered) or HBM hash-table
// (unordered) kernels of k_flat.cu for that batch instead.
#include "mm_kernels.h"
#include "mm_smem.cuh"

namespace mm {

// Bucket hash: Fibonacci (multiply-shift) hashing of the 64-bit tuple -- a
// handful of instructions instead of three Jenkins rounds, and independent of
// mm_route's owner hash (Jenkins), so the shard a rank owns still spreads over
// all buckets.
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

// Buckets: B = 2^nb with at most `avg` elements of the larger side per
// bucket on average; each bucket owns a fixed region of 3 avg slots per side
// (a bucket above it -- heavily repeated tuples -- flags an overflow).  The
// geometry is per level (bucket_avg): NOWILD_ORDERED 256 elements per side
// with 128-thread CTAs, six per SM; NOWILD_UNORDERED 512 with 256-thread
// CTAs, three per SM (A/B).
#ifndef MM_UNORD_AVG
#define MM_UNORD_AVG 512  // A/B: NOWILD_UNORDERED bucket geometry (512: 256 threads x 3 CTAs, 256: 128 x 6)
#endif
int bucket_avg(bool ordered) { return ordered ? 256 : MM_UNORD_AVG; }

int bucket_bits_for(int64_t n_side, int avg) {
  int nb = 1;
  while (nb < 30 && ((int64_t)1 << nb) * avg < n_side) nb++;
  return nb;
}
int64_t bucket_count(int64_t n_side, int avg) { return (int64_t)1 << bucket_bits_for(n_side, avg); }

// ------------------------------------------------------------- partition
// MSD passes over the bucket id b = bucket_of(hdr) (nb bits): pass 0 reads
// the snapshot and splits each side by the top bits of b, every later pass
// splits each region of the previous one by the next bits; the last pass
// writes the buckets' 3 avg-slot regions.  Every region has a fixed
// capacity (the expected size x 1.25 + 256 on intermediate levels), so a
// pass needs no histogram pass and no scan: a tile of kPassTile elements
// ranks its elements per digit with shared-memory atomics, reserves each
// digit's run in the child region with ONE global atomic, stages the tile in
// digit order in shared memory and writes every run with consecutive threads
// (coalesced).  The order inside a region is not the snapshot order; the
// snapshot index travels with the header and the matching kernel orders
// equal tuples by it where order matters.  Reads 8 B (pass 0) or 12 B and
// writes 12 B per element and pass.
#ifndef MM_PASS_THREADS
#define MM_PASS_THREADS 512  // A/B (tools/gpu_ab_pass.sh): 512 x 8 x 2 CTAs/SM beats 256 x 8/16, 1024 x 4/8, 512 x 4/16
#endif
#ifndef MM_PASS_ITEMS
#define MM_PASS_ITEMS 8
#endif
#ifndef MM_UNORD_POP
#define MM_UNORD_POP 1  // A/B: NOWILD_UNORDERED buckets matched by tuple stacks (k_bucket_pop; configs[3] 17.45 -> 20.17 G/s)
#endif
#ifndef MM_PASS_VEC
#define MM_PASS_VEC 1  // A/B: later passes load element pairs with vector loads
#endif
#ifndef MM_PASS_MINB
#define MM_PASS_MINB 2
#endif
constexpr int kPassThreads = MM_PASS_THREADS;
constexpr int kPassItems = MM_PASS_ITEMS;
constexpr int kPassTile = kPassThreads * kPassItems;  // 4096
constexpr int kPassMaxKeys = 1024;                    // digits per tile (pass 0: both sides' digits)

PartPlan part_plan(int64_t n_side, int avg) {
  PartPlan pl{};
  pl.nb = bucket_bits_for(n_side, avg);
  // pass 0 takes at most 8 bits (2 x 256 keys per tile), later passes at most 10
  int rest = pl.nb;
  int bits[kMaxPasses];
  int np = 0;
  // two passes up to nb = 19 (9 + 10 bits: 2 x 512 keys, then 1024 keys per
  // tile), three beyond
  const int first = rest <= 8 ? rest : (rest <= 18 ? rest - rest / 2 : (rest == 19 ? 9 : 8));  // <= 9: 2 x 512 keys
  bits[np++] = first;
  rest -= first;
  const int later = (rest + 9) / 10;  // fewest later passes of <= 10 bits, bits spread evenly
  for (int i = 0; i < later; i++) {
    const int b = (rest + (later - i) - 1) / (later - i);
    bits[np++] = b;
    rest -= b;
  }
  pl.passes = np;
  int done = 0;
  int64_t off = 0;
  for (int i = 0; i < np; i++) {
    done += bits[i];
    pl.bits[i] = bits[i];
    pl.shift[i] = pl.nb - done;
    pl.children[i] = (int64_t)1 << done;  // per side
    if (i == np - 1) {
      pl.cap[i] = 3 * avg;
    } else {
      const int64_t expect = (n_side + pl.children[i] - 1) / pl.children[i];
      pl.cap[i] = (expect + expect / 4 + 256 + 15) / 16 * 16;
    }
    pl.cnt_off[i] = off;
    off += 2 * pl.children[i];
    pl.slots[i] = pl.children[i] * pl.cap[i];
  }
  pl.cnt_total = off;
  // intermediate levels alternate between two scratch buffers
  pl.scratch_slots[0] = pl.scratch_slots[1] = 0;
  for (int i = 0; i + 1 < np; i++)
    if (pl.slots[i] > pl.scratch_slots[i & 1]) pl.scratch_slots[i & 1] = pl.slots[i];
  return pl;
}

struct PassArgs {
  // input: pass 0 the snapshot (receives [0, n0), messages [n0, n)); later
  // passes the regions of the previous level (P parents per side)
  SnapRead snap[2];
  int64_t n0, n;
  const uint64_t* ih[2];
  const uint32_t* iix[2];
  const uint32_t* icnt;  // [2][P]
  int64_t icap;
  uint32_t P;
  uint32_t tiles_per_parent;
  // output: P x F children per side
  uint64_t* oh[2];
  uint32_t* oix[2];
  uint32_t* ocnt;  // [2][P F]
  int64_t ocap;
  int nb, shift, fbits;
  uint32_t* overflow;
};

struct PassSmem {
  uint64_t h[kPassTile];
  uint32_t ix[kPassTile];
  uint16_t key[kPassTile];
  uint32_t hist[kPassMaxKeys];
  uint32_t lstart[kPassMaxKeys];
  uint32_t gbase[kPassMaxKeys];
  uint32_t scan_sm[kPassThreads / 32 + 1];
};

template <bool FIRST>
__global__ void __launch_bounds__(kPassThreads, MM_PASS_MINB) k_part_pass(PassArgs a) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  PassSmem& sm = *reinterpret_cast<PassSmem*>(smem_raw);
  const int tid = threadIdx.x;
  const uint32_t F = 1u << a.fbits;
  const uint32_t nkeys = FIRST ? 2 * F : F;
  // the tile: pass 0 -- elements [t0, t1) of the concatenated sides;
  // later passes -- side sd, parent p, elements [t0, t1) of its region
  int sd = 0;
  uint32_t parent = 0;
  int64_t t0, t1;
  if (FIRST) {
    t0 = (int64_t)blockIdx.x * kPassTile;
    t1 = t0 + kPassTile < a.n ? t0 + kPassTile : a.n;
  } else {
    const uint32_t pt = blockIdx.x / a.tiles_per_parent;  // side * P + parent
    sd = pt >= a.P;
    parent = pt - (sd ? a.P : 0);
    const int64_t c = a.icnt[pt] < (uint32_t)a.icap ? a.icnt[pt] : (uint32_t)a.icap;
    t0 = (int64_t)(blockIdx.x % a.tiles_per_parent) * kPassTile;
    t1 = t0 + kPassTile < c ? t0 + kPassTile : c;
  }
  if (t0 >= t1) return;  // uniform
  for (uint32_t k = tid; k < nkeys; k += kPassThreads) sm.hist[k] = 0;
  __syncthreads();
  uint64_t h[kPassItems];
  uint32_t ix[kPassItems], key[kPassItems], rank[kPassItems];
  const int64_t rbase = FIRST ? 0 : (int64_t)parent * a.icap;
  // element of item u: later passes read pairs of consecutive elements with
  // one 16-byte (headers) and one 8-byte (indices) load (MM_PASS_VEC); the
  // order inside a digit run is free, so any mapping of elements to threads
  // is valid
  auto elem = [&](int u) -> int64_t {
    if (!FIRST && MM_PASS_VEC) return t0 + (int64_t)(u >> 1) * (2 * kPassThreads) + 2 * tid + (u & 1);
    return t0 + (int64_t)u * kPassThreads + tid;
  };
  if (!FIRST && MM_PASS_VEC) {
    const uint64_t* ih = (sd ? a.ih[1] : a.ih[0]) + rbase;
    const uint32_t* iix = (sd ? a.iix[1] : a.iix[0]) + rbase;
#pragma unroll
    for (int v = 0; v < kPassItems / 2; v++) {  // every load in flight first
      const int64_t k = elem(2 * v);
      if (k + 1 < t1) {
        const ulonglong2 hh = *reinterpret_cast<const ulonglong2*>(ih + k);
        const uint2 xx = *reinterpret_cast<const uint2*>(iix + k);
        h[2 * v] = hh.x;
        h[2 * v + 1] = hh.y;
        ix[2 * v] = xx.x;
        ix[2 * v + 1] = xx.y;
      } else if (k < t1) {
        h[2 * v] = ih[k];
        ix[2 * v] = iix[k];
      }
    }
  } else {
#pragma unroll
    for (int u = 0; u < kPassItems; u++) {  // every load in flight first
      const int64_t k = elem(u);
      if (k < t1) {
        if (FIRST) {
          const bool m = k >= a.n0;
          ix[u] = (uint32_t)(m ? k - a.n0 : k);
          h[u] = m ? a.snap[1].hdr(ix[u]) : a.snap[0].hdr(ix[u]);
        } else {
          h[u] = (sd ? a.ih[1] : a.ih[0])[rbase + k];
          ix[u] = (sd ? a.iix[1] : a.iix[0])[rbase + k];
        }
      }
    }
  }
#pragma unroll
  for (int u = 0; u < kPassItems; u++) {
    const int64_t k = elem(u);
    if (k < t1) {
      const uint32_t d = (bucket_of(h[u], a.nb) >> a.shift) & (F - 1);
      key[u] = FIRST ? (k >= a.n0 ? F + d : d) : d;
      rank[u] = atomicAdd(&sm.hist[key[u]], 1u);
    }
  }
  __syncthreads();
  // tile-local digit starts (block scan) and one global reservation per digit
  {
    constexpr int KPT = kPassMaxKeys / kPassThreads;
    uint32_t v[KPT], sum = 0;
#pragma unroll
    for (int j = 0; j < KPT; j++) {
      const uint32_t k = tid * KPT + j;
      v[j] = k < nkeys ? sm.hist[k] : 0u;
      sum += v[j];
    }
    uint32_t all;
    uint32_t ex = block_excl_scan<uint32_t>(sum, sm.scan_sm, &all);
#pragma unroll
    for (int j = 0; j < KPT; j++) {
      const uint32_t k = tid * KPT + j;
      if (k < nkeys) {
        sm.lstart[k] = ex;
        if (v[j]) {
          const uint32_t side = FIRST ? (k >= F) : (uint32_t)sd;
          const uint32_t child = FIRST ? (k >= F ? k - F : k) : parent * F + k;
          const int64_t nchild = FIRST ? F : (int64_t)a.P * F;
          sm.gbase[k] = atomicAdd(&a.ocnt[side * nchild + child], v[j]);
        }
      }
      ex += v[j];
    }
  }
  __syncthreads();
#pragma unroll
  for (int u = 0; u < kPassItems; u++) {
    const int64_t k = elem(u);
    if (k < t1) {
      const uint32_t pos = sm.lstart[key[u]] + rank[u];
      sm.h[pos] = h[u];
      sm.ix[pos] = ix[u];
      sm.key[pos] = (uint16_t)key[u];
    }
  }
  __syncthreads();
  const uint32_t tn = (uint32_t)(t1 - t0);
  for (uint32_t p = tid; p < tn; p += kPassThreads) {
    const uint32_t k = sm.key[p];
    const uint32_t off = sm.gbase[k] + (p - sm.lstart[k]);
    const uint32_t side = FIRST ? (k >= F) : (uint32_t)sd;
    const uint32_t child = FIRST ? (k >= F ? k - F : k) : parent * F + k;
    if (off < (uint32_t)a.ocap) {
      const int64_t dst = (int64_t)child * a.ocap + off;
      (side ? a.oh[1] : a.oh[0])[dst] = sm.h[p];
      (side ? a.oix[1] : a.oix[0])[dst] = sm.ix[p];
    } else if (off == (uint32_t)a.ocap) {
      atomicOr(a.overflow, 1u);
    }
  }
}

// Output offsets of the buckets: exclusive scan of the receive counts.
struct BucketCountIn {
  const uint32_t* cnt;
  uint32_t cap;
  __device__ __forceinline__ uint32_t operator()(int64_t b) const {
    const uint32_t c = cnt[b];
    return c < cap ? c : cap;
  }
};
struct BucketOffOut {
  uint32_t* off;
  int64_t B;
  __device__ __forceinline__ void operator()(int64_t b, uint32_t ex, uint32_t v) const {
    off[b] = ex;
    if (b == B - 1) off[B] = ex + v;
  }
};

// ------------------------------------------------------------ matching kernel
// One bucket per CTA iteration (persistent grid), entirely in shared memory:
//  A  the bucket's receives [0, nr) and messages [nr, nr + nm) are loaded;
//  B  every tuple gets a dense id from an open-addressing table of 32-bit
//     entries (16-bit fingerprint | representative element; the CAS winner
//     draws the id);
//  C  per tuple, receives and messages are counted with one packed 16|16
//     shared atomic each, which also gives every element a position among
//     its side's equal tuples;
//  D  one block scan of the packed counts: each tuple's group start in the
//     receive area and in the message area;
//  E  elements placed by (tuple, position);
//  F  NOWILD_ORDERED only: each group re-ordered by snapshot index (an
//     element's rank = the group members with a smaller index; groups are a
//     few elements), so the group is in posting / arrival order;
//  G  the receive at group position j takes the message at group position j
//     (the n-th receive of a tuple takes the n-th message: PAPER.md §VI.A;
//     for NOWILD_UNORDERED any maximal pairing, §VI.C l.215), results are
//     written coalesced at the bucket's output offset in group order, and a
//     matched byte per bucket slot (coalesced) serves a later compaction.
// O(1) shared-memory work per element (F: O(group size)), 7 barriers.
constexpr uint32_t kNone32 = 0xFFFFFFFFu;

// Shared memory of one bucket of up to K = 4 avg elements (receives +
// messages) and H = 8 avg table slots: 32 B per element (avg 512: 64 KB,
// three CTAs per SM; avg 256: 32 KB, six).  Arrays that die with a phase
// share space with arrays that start later.
template <int K, int H, int NT>
struct MatchSmem {
  union {
    uint64_t hdr[K];  // A..B: headers (table keys)
    struct {
      uint32_t aidx[K];  // E..F: snapshot index of each grouped element
      uint16_t srt[K];   // F..G: every group in snapshot order
    };
  };
  union {
    uint32_t table[H];  // A..B: (fingerprint << 16) | representative element
    uint16_t area[K];   // E..F: receives [0, nr) then messages [nr, n), grouped by tuple
  };
  uint32_t idx[K];      // snapshot index
  uint16_t sid[H];      // B..C: slot -> dense tuple id
  uint16_t tup[K];      // B: element -> slot; C..: tuple id
  uint16_t pos[K];      // C..E: position among its side's equal tuples
  uint32_t pre[K + 1];  // C: packed counts (#recv | #msg << 16); D..: packed group starts, pre[T] = totals
  uint32_t wsum[NT / 32];
  uint32_t ntup;
  uint32_t nmatch;
};
static_assert(sizeof(MatchSmem<2048, 4096, 256>) <= 74 * 1024, "avg 512: three CTAs per SM");
static_assert(sizeof(MatchSmem<1024, 2048, 128>) <= 37 * 1024, "avg 256: six CTAs per SM");

struct MatchArgs {
  FlatArgs a;
  const uint64_t* h[2];
  const uint32_t* ix[2];
  const uint32_t* cnt;  // [2][B]
  const uint32_t* roff;  // [B + 1] output offsets
  uint8_t* sflag[2];     // matched byte per bucket slot
  uint32_t* overflow;
  uint32_t B;
};

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

template <bool ORDERED, int AVG, int NT, int MINB>
__global__ void __launch_bounds__(NT, MINB) k_bucket_match(MatchArgs ma) {
  constexpr int kMatchK = 4 * AVG;            // receives + messages of one bucket on chip
  constexpr uint32_t kMatchH = 8 * AVG;       // table slots (>= 2 kMatchK)
  constexpr uint32_t kSideCap = 3 * AVG;      // region slots per side
  extern __shared__ __align__(16) uint8_t smem_raw[];
  auto& sm = *reinterpret_cast<MatchSmem<kMatchK, kMatchH, NT>*>(smem_raw);
  constexpr int PER = kMatchK / NT;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t lt = lanemask_lt();
  const FlatArgs& a = ma.a;
  const int64_t rres = a.R.q_len[0], rpb = a.R.pend_begin(0);
  const int64_t mres = a.M.q_len[0], mpb = a.M.pend_begin(0);
  constexpr uint32_t hmask = kMatchH - 1;
  // Persistent: buckets blockIdx.x, + G, ...; the next bucket's elements are
  // loaded into registers while the current one is matched, and the counts of
  // the one after that are loaded a bucket ahead of its elements.
  const uint32_t G = gridDim.x;
  uint64_t hv[PER];
  uint32_t iv[PER];
  auto counts = [&](uint32_t bb, uint32_t& fnr, uint32_t& fnm) {
    fnr = fnm = 0;
    if (bb < ma.B) {
      fnr = ma.cnt[bb];
      fnm = ma.cnt[ma.B + bb];
    }
  };
  auto fetch = [&](uint32_t bb, uint32_t fnr, uint32_t fnm) {
    const bool fits = fnr <= kSideCap && fnm <= kSideCap && fnr + fnm <= (uint32_t)kMatchK;
    const int64_t base = (int64_t)bb * kSideCap;
#pragma unroll
    for (int u = 0; u < PER; u++) {
      const uint32_t e = tid + u * NT;
      hv[u] = 0;
      iv[u] = 0;
      if (fits && e < fnr) {
        hv[u] = ma.h[0][base + e];
        iv[u] = ma.ix[0][base + e];
      } else if (fits && e < fnr + fnm) {
        hv[u] = ma.h[1][base + e - fnr];
        iv[u] = ma.ix[1][base + e - fnr];
      }
    }
  };
  uint32_t xnr, xnm, ynr, ynm;  // sizes of the bucket held in hv / iv, and of the next one
#ifdef MM_PHASE_TIMING
  long long t_bphase = clock64();
#endif
  counts(blockIdx.x, xnr, xnm);
  fetch(blockIdx.x, xnr, xnm);
  counts(blockIdx.x + G, ynr, ynm);
  for (uint32_t b = blockIdx.x; b < ma.B; b += G) {
    __syncthreads();  // the previous bucket is done with shared memory
    MM_BPHASE(0);
    const uint32_t nr = xnr, nm = xnm, n = nr + nm;
    if (n == 0 || nr > kSideCap || nm > kSideCap || n > (uint32_t)kMatchK) {  // uniform across the CTA
      if (n > (uint32_t)kMatchK && tid == 0) atomicOr(ma.overflow, 1u);
      xnr = ynr;
      xnm = ynm;
      fetch(b + G, xnr, xnm);
      counts(b + 2 * G, ynr, ynm);
      continue;
    }
    // A: registers to shared memory, clear the table, prefetch
#pragma unroll
    for (int u = 0; u < PER; u++) {
      const uint32_t e = tid + u * NT;
      if (e < n) {
        sm.hdr[e] = hv[u];
        sm.idx[e] = iv[u];
      }
    }
    for (uint32_t s = tid; s < kMatchH / 4; s += NT) reinterpret_cast<uint4*>(sm.table)[s] = make_uint4(~0u, ~0u, ~0u, ~0u);
    if (tid == 0) {
      sm.ntup = 0;
      sm.nmatch = 0;
    }
    xnr = ynr;
    xnm = ynm;
    fetch(b + G, xnr, xnm);
    counts(b + 2 * G, ynr, ynm);
    __syncthreads();
    MM_BPHASE(1);
    // B: every tuple into the table; the CAS winners of a warp draw their
    // dense ids with one atomic and zero their counters
    for (uint32_t e0 = warp * 32; e0 < n; e0 += NT) {
      const uint32_t e = e0 + lane;
      bool won = false;
      uint32_t s = 0;
      if (e < n) {
        const uint64_t h = sm.hdr[e];
        const uint64_t p = h * 0xD6E8FEB86659FD93ull;
        s = (uint32_t)(p >> 40) & hmask;
        const uint32_t fp = (uint32_t)(p >> 24) & 0xFFFFu;
        while (true) {
          uint32_t o = sm.table[s];
          if (o == 0xFFFFFFFFu) {
            o = atomicCAS(&sm.table[s], 0xFFFFFFFFu, (fp << 16) | e);  // representative's header is in smem already
            if (o == 0xFFFFFFFFu) {
              won = true;
              break;
            }
          }
          if ((o >> 16) == fp && sm.hdr[o & 0xFFFFu] == h) break;
          s = (s + 1) & hmask;
        }
        sm.tup[e] = (uint16_t)s;
      }
      const uint32_t wm = __ballot_sync(kFull, won);
      uint32_t base = 0;
      if (lane == 0 && wm) base = atomicAdd(&sm.ntup, (uint32_t)__popc(wm));
      base = __shfl_sync(kFull, base, 0);
      if (won) {
        const uint32_t id = base + __popc(wm & lt);
        sm.sid[s] = (uint16_t)id;
        sm.pre[id] = 0;
      }
    }
    __syncthreads();
    MM_BPHASE(2);
    // C: tuple ids; per tuple, receives count in the low and messages in the
    // high half of one word -- the old value is the element's position
    for (uint32_t e = tid; e < n; e += NT) {
      const uint32_t t = sm.sid[sm.tup[e]];
      sm.tup[e] = (uint16_t)t;
      const bool msg = e >= nr;
      const uint32_t old = atomicAdd(&sm.pre[t], msg ? 0x10000u : 1u);
      sm.pos[e] = (uint16_t)(msg ? old >> 16 : old & 0xFFFFu);
    }
    __syncthreads();
    MM_BPHASE(3);
    // D: group starts = exclusive scan of the packed counts (no carry: both
    // halves stay below kMatchK); one barrier -- warp totals, then every
    // thread adds the totals of the warps before it
    const uint32_t T = sm.ntup;
    {
      uint32_t v[PER], sum = 0;
#pragma unroll
      for (int j = 0; j < PER; j++) {
        const uint32_t t = PER * tid + j;
        v[j] = t < T ? sm.pre[t] : 0u;
        sum += v[j];
      }
      uint32_t inc = sum;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t x = __shfl_up_sync(kFull, inc, o);
        if (lane >= o) inc += x;
      }
      if (lane == 31) sm.wsum[warp] = inc;
      __syncthreads();
      uint32_t ex = inc - sum, all = 0;
#pragma unroll
      for (int w = 0; w < NT / 32; w++) {
        const uint32_t x = sm.wsum[w];
        ex += w < warp ? x : 0u;
        all += x;
      }
#pragma unroll
      for (int j = 0; j < PER; j++) {
        const uint32_t t = PER * tid + j;
        if (t < T) sm.pre[t] = ex;
        ex += v[j];
      }
      if (tid == 0) sm.pre[T] = all;
    }
    __syncthreads();
    MM_BPHASE(4);
    // E: placement by (tuple, position)
    for (uint32_t e = tid; e < n; e += NT) {
      const uint32_t t = sm.tup[e], p = sm.pre[t];
      const uint32_t slot = e >= nr ? nr + (p >> 16) + sm.pos[e] : (p & 0xFFFFu) + sm.pos[e];
      sm.area[slot] = (uint16_t)e;
      if (ORDERED) sm.aidx[slot] = sm.idx[e];
    }
    __syncthreads();
    MM_BPHASE(5);
    const uint16_t* grp = sm.area;
    if (ORDERED) {
      // F: each group in snapshot order -- the rank of an element is the
      // number of its group's members with a smaller snapshot index
      for (uint32_t x = tid; x < n; x += NT) {
        const uint32_t e = sm.area[x];
        const uint32_t t = sm.tup[e], p = sm.pre[t], c = sm.pre[t + 1] - p;
        const bool msg = x >= nr;
        const uint32_t g0 = msg ? nr + (p >> 16) : (p & 0xFFFFu);
        const uint32_t gn = msg ? (c >> 16) : (c & 0xFFFFu);
        const uint32_t my = sm.aidx[x];
        uint32_t rank = 0;
        for (uint32_t y = g0; y < g0 + gn; y++) rank += sm.aidx[y] < my;
        sm.srt[g0 + rank] = (uint16_t)e;
      }
      __syncthreads();
      MM_BPHASE(6);
      grp = sm.srt;
    }
    // G: the receive at group position j takes the message at position j
    const int64_t obase = ma.roff[b];
    const int64_t sbase = (int64_t)b * kSideCap;
    uint32_t nmatch = 0;
    for (uint32_t s = tid; s < n; s += NT) {
      const uint32_t e = grp[s];
      const uint32_t t = sm.tup[e], p = sm.pre[t], c = sm.pre[t + 1] - p;
      if (s < nr) {
        const uint32_t j = s - (p & 0xFFFFu);
        int64_t mc = MM_NO_MATCH;
        if (j < (c >> 16)) {
          const uint32_t m = grp[nr + (p >> 16) + j];
          mc = a.M.cookie(0, sm.idx[m], mres, mpb);
          nmatch++;
        }
        a.out_rc[obase + s] = a.R.cookie(0, sm.idx[e], rres, rpb);
        a.out_mc[obase + s] = mc;
        ma.sflag[0][sbase + e] = mc != MM_NO_MATCH;
      } else {
        const uint32_t j = s - nr - (p >> 16);
        ma.sflag[1][sbase + (e - nr)] = j < (c & 0xFFFFu);
      }
    }
    for (int o = 16; o; o >>= 1) nmatch += __shfl_xor_sync(kFull, nmatch, o);
    if (lane == 0 && nmatch) atomicAdd(&sm.nmatch, nmatch);
    __syncthreads();
    if (tid == 0 && sm.nmatch) atomicAdd(a.n_matched, (unsigned long long)sm.nmatch);
    MM_BPHASE(7);
#ifdef MM_PHASE_TIMING
    if (tid == 0) atomicAdd(&g_bucket_cycles[15], 1ull);
#endif
  }
}

// NOWILD_UNORDERED, stack variant (MM_UNORD_POP): any maximal pairing of
// equal tuples needs no grouping, so a bucket is matched with three
// barriers instead of seven: B every element enters the table (the CAS
// winner's element represents the tuple; losers compare with its header
// in shared memory), every message pushes itself on its tuple's stack
// (atomicExch on the slot word); C every receive draws a ticket p from the
// same word (atomicAdd of 1 << 16: the old word also holds the stack head)
// and takes the stack's p-th message, if any (a walk of p links -- groups
// are a few elements; a tuple with kPopWalk or more receives has its stack
// laid out flat once and its later receives index it: no run-length limit);
// D the messages' matched flags are written coalesced.
// Receives are reported in bucket order (any order is allowed, mm.h).
constexpr uint32_t kPopWalk = 64;

template <int K, int H, int NT>
struct PopSmem {
  uint64_t hdr[K];    // A..B; then (as uint16) deep tuples' stacks laid out flat
  uint32_t idx[K];
  uint32_t table[H];  // (fingerprint << 16) | representative element
  uint32_t hw[H];     // (receive tickets << 16) | message stack head
  uint16_t nxt[K];    // message -> next message of its tuple's stack; deep receive -> its ticket
  uint16_t slot[K];   // receive -> its tuple's slot
  uint32_t mbits[K / 32];
  uint32_t dbits[K / 32];  // deep receives (ticket >= kPopWalk)
  uint32_t nmatch;
  uint32_t deep, ftop;
};

template <int AVG, int NT, int MINB>
__global__ void __launch_bounds__(NT, MINB) k_bucket_pop(MatchArgs ma) {
  constexpr int kK = 4 * AVG;
  constexpr uint32_t kH = 8 * AVG;
  constexpr uint32_t kSideCap = 3 * AVG;
  extern __shared__ __align__(16) uint8_t smem_raw[];
  auto& sm = *reinterpret_cast<PopSmem<kK, kH, NT>*>(smem_raw);
  constexpr int PER = kK / NT;
  const int tid = threadIdx.x, lane = tid & 31;
  const FlatArgs& a = ma.a;
  const int64_t rres = a.R.q_len[0], rpb = a.R.pend_begin(0);
  const int64_t mres = a.M.q_len[0], mpb = a.M.pend_begin(0);
  constexpr uint32_t hmask = kH - 1;
  const uint32_t G = gridDim.x;
  uint64_t hv[PER];
  uint32_t iv[PER];
  auto counts = [&](uint32_t bb, uint32_t& fnr, uint32_t& fnm) {
    fnr = fnm = 0;
    if (bb < ma.B) {
      fnr = ma.cnt[bb];
      fnm = ma.cnt[ma.B + bb];
    }
  };
  auto fetch = [&](uint32_t bb, uint32_t fnr, uint32_t fnm) {
    const bool fits = fnr <= kSideCap && fnm <= kSideCap && fnr + fnm <= (uint32_t)kK;
    const int64_t base = (int64_t)bb * kSideCap;
#pragma unroll
    for (int u = 0; u < PER; u++) {
      const uint32_t e = tid + u * NT;
      hv[u] = 0;
      iv[u] = 0;
      if (fits && e < fnr) {
        hv[u] = ma.h[0][base + e];
        iv[u] = ma.ix[0][base + e];
      } else if (fits && e < fnr + fnm) {
        hv[u] = ma.h[1][base + e - fnr];
        iv[u] = ma.ix[1][base + e - fnr];
      }
    }
  };
  uint32_t xnr, xnm, ynr, ynm;
  counts(blockIdx.x, xnr, xnm);
  fetch(blockIdx.x, xnr, xnm);
  counts(blockIdx.x + G, ynr, ynm);
  for (uint32_t b = blockIdx.x; b < ma.B; b += G) {
    __syncthreads();  // the previous bucket is done with shared memory
    const uint32_t nr = xnr, nm = xnm, n = nr + nm;
    if (n == 0 || nr > kSideCap || nm > kSideCap || n > (uint32_t)kK) {  // uniform across the CTA
      if (n > (uint32_t)kK && tid == 0) atomicOr(ma.overflow, 1u);
      xnr = ynr;
      xnm = ynm;
      fetch(b + G, xnr, xnm);
      counts(b + 2 * G, ynr, ynm);
      continue;
    }
    // A: registers to shared memory, tables cleared, next bucket prefetched
#pragma unroll
    for (int u = 0; u < PER; u++) {
      const uint32_t e = tid + u * NT;
      if (e < n) {
        sm.hdr[e] = hv[u];
        sm.idx[e] = iv[u];
      }
    }
    for (uint32_t x = tid; x < kH / 4; x += NT) {
      reinterpret_cast<uint4*>(sm.table)[x] = make_uint4(~0u, ~0u, ~0u, ~0u);
      reinterpret_cast<uint4*>(sm.hw)[x] = make_uint4(0xFFFFu, 0xFFFFu, 0xFFFFu, 0xFFFFu);
    }
    for (uint32_t x = tid; x < kK / 32; x += NT) {
      sm.mbits[x] = 0u;
      sm.dbits[x] = 0u;
    }
    if (tid == 0) {
      sm.nmatch = 0;
      sm.deep = 0;
      sm.ftop = 0;
    }
    xnr = ynr;
    xnm = ynm;
    fetch(b + G, xnr, xnm);
    counts(b + 2 * G, ynr, ynm);
    __syncthreads();
    // B: tuples into the table; messages onto their tuple's stack
    for (uint32_t e = tid; e < n; e += NT) {
      const uint64_t h = sm.hdr[e];
      const uint64_t pr = h * 0xD6E8FEB86659FD93ull;
      uint32_t sl = (uint32_t)(pr >> 40) & hmask;
      const uint32_t fp = (uint32_t)(pr >> 24) & 0xFFFFu;
      while (true) {
        uint32_t o = sm.table[sl];
        if (o == 0xFFFFFFFFu) {
          o = atomicCAS(&sm.table[sl], 0xFFFFFFFFu, (fp << 16) | e);  // the representative's header is in smem
          if (o == 0xFFFFFFFFu) break;
        }
        if ((o >> 16) == fp && sm.hdr[o & 0xFFFFu] == h) break;
        sl = (sl + 1) & hmask;
      }
      if (e >= nr) sm.nxt[e] = (uint16_t)(atomicExch(&sm.hw[sl], e) & 0xFFFFu);
      else sm.slot[e] = (uint16_t)sl;
    }
    __syncthreads();
    // C: every receive draws a ticket on its tuple's stack
    const int64_t obase = ma.roff[b];
    const int64_t sbase = (int64_t)b * kSideCap;
    uint32_t nmatch = 0;
    auto emit = [&](uint32_t r, uint32_t m) {
      int64_t mc = MM_NO_MATCH;
      if (m != 0xFFFFu) {
        mc = a.M.cookie(0, sm.idx[m], mres, mpb);
        atomicOr(&sm.mbits[(m - nr) >> 5], 1u << ((m - nr) & 31u));
        nmatch++;
      }
      a.out_rc[obase + r] = a.R.cookie(0, sm.idx[r], rres, rpb);
      a.out_mc[obase + r] = mc;
      ma.sflag[0][sbase + r] = m != 0xFFFFu;
    };
    for (uint32_t r = tid; r < nr; r += NT) {
      const uint32_t old = atomicAdd(&sm.hw[sm.slot[r]], 0x10000u);
      uint32_t p = old >> 16, m = old & 0xFFFFu;
      if (p >= kPopWalk) {  // a deep tuple: resolved below from its flattened stack
        sm.nxt[r] = (uint16_t)p;
        atomicOr(&sm.dbits[r >> 5], 1u << (r & 31u));
        sm.deep = 1u;
        continue;
      }
      while (p > 0 && m != 0xFFFFu) {
        m = sm.nxt[m];
        p--;
      }
      emit(r, m);
    }
    for (int o = 16; o; o >>= 1) nmatch += __shfl_xor_sync(kFull, nmatch, o);
    if (lane == 0 && nmatch) atomicAdd(&sm.nmatch, nmatch);
    nmatch = 0;
    __syncthreads();
    if (sm.deep) {  // (uniform) tuples with >= kPopWalk receives: no run-length limit
      uint16_t* flat = reinterpret_cast<uint16_t*>(sm.hdr);  // the headers are dead after B
      // the receive holding ticket kPopWalk flattens its tuple's message stack
      // once; the table entry (dead after B) keeps the flat array's base | length
      for (uint32_t r = tid; r < nr; r += NT)
        if (((sm.dbits[r >> 5] >> (r & 31u)) & 1u) && sm.nxt[r] == kPopWalk) {
          uint32_t len = 0;
          for (uint32_t x = sm.hw[sm.slot[r]] & 0xFFFFu; x != 0xFFFFu; x = sm.nxt[x]) len++;
          const uint32_t base = atomicAdd(&sm.ftop, len);
          uint32_t q = base;
          for (uint32_t x = sm.hw[sm.slot[r]] & 0xFFFFu; x != 0xFFFFu; x = sm.nxt[x]) flat[q++] = (uint16_t)x;
          sm.table[sm.slot[r]] = base | (len << 16);
        }
      __syncthreads();
      for (uint32_t r = tid; r < nr; r += NT)
        if ((sm.dbits[r >> 5] >> (r & 31u)) & 1u) {
          const uint32_t t = sm.table[sm.slot[r]], p = sm.nxt[r];
          emit(r, p < (t >> 16) ? (uint32_t)flat[(t & 0xFFFFu) + p] : 0xFFFFu);
        }
      if (nmatch) atomicAdd(&sm.nmatch, nmatch);
      __syncthreads();
    }
    // D: the messages' matched flags
    for (uint32_t j = tid; j < nm; j += NT) ma.sflag[1][sbase + j] = (sm.mbits[j >> 5] >> (j & 31u)) & 1u;
    if (tid == 0 && sm.nmatch) atomicAdd(a.n_matched, (unsigned long long)sm.nmatch);
  }
}

template <auto KERNEL>
static uint32_t persistent_grid(int threads, size_t smem, uint32_t B) {
  const uint32_t g = (uint32_t)resident_ctas<KERNEL>(threads, smem);
  return g < B ? g : B;
}

// Largest allocation any batch of at most n_side elements per side needs.
PartPlan part_plan_alloc(int64_t n_side, int avg) {
  PartPlan m = part_plan(n_side, avg);
  for (int nb = 1; nb < m.nb; nb++) {
    const PartPlan p = part_plan(((int64_t)1 << nb) * avg, avg);
    for (int j = 0; j < 2; j++)
      if (p.scratch_slots[j] > m.scratch_slots[j]) m.scratch_slots[j] = p.scratch_slots[j];
    if (p.cnt_total > m.cnt_total) m.cnt_total = p.cnt_total;
  }
  return m;
}

// One bucket geometry's matching kernel: avg elements per side and bucket,
// NT threads, MINB CTAs per SM.
template <bool ORDERED, int AVG, int NT, int MINB>
static cudaError_t launch_bucket_match(const MatchArgs& ma, uint32_t B, cudaStream_t st) {
  constexpr auto kern = k_bucket_match<ORDERED, AVG, NT, MINB>;
  const size_t smem = sizeof(MatchSmem<4 * AVG, 8 * AVG, NT>);
  cudaError_t err = ensure_dyn_smem<kern>(smem);
  if (err != cudaSuccess) return err;
  count_launch();
  kern<<<persistent_grid<kern>(NT, smem, B), NT, smem, st>>>(ma);
  return cudaGetLastError();
}

cudaError_t run_bucketed(const FlatArgs& a, bool ordered, BucketScratch& s, cudaStream_t st) {
  const int avg = bucket_avg(ordered);
  const PartPlan pl = part_plan(a.nr > a.nm ? a.nr : a.nm, avg);
  s.side_cap = 3 * avg;
  const int nb = pl.nb;
  const uint32_t B = 1u << nb;
  s.plan = pl;
  s.B = B;
  const int last = pl.passes - 1;
  s.bcnt = s.cnt + pl.cnt_off[last];
  s.overflow = s.cnt + pl.cnt_total;  // cleared with the counts (one memset)
  cudaError_t err;
  if ((err = cudaMemsetAsync(s.cnt, 0, sizeof(uint32_t) * (pl.cnt_total + 1), st)) != cudaSuccess) return err;
  PassArgs pa{};
  pa.snap[0] = SnapRead{a.R.q_hdr, a.R.p_hdr, s.rres};
  pa.snap[1] = SnapRead{a.M.q_hdr, a.M.p_hdr, s.mres};
  pa.n0 = a.nr;
  pa.n = a.nr + a.nm;
  pa.nb = nb;
  pa.overflow = s.overflow;
  const size_t psmem = sizeof(PassSmem);
  for (int i = 0; i < pl.passes && pa.n > 0; i++) {
    pa.fbits = pl.bits[i];
    pa.shift = pl.shift[i];
    pa.ocap = pl.cap[i];
    pa.ocnt = s.cnt + pl.cnt_off[i];
    for (int sd = 0; sd < 2; sd++) {
      pa.oh[sd] = i == last ? s.h[sd] : s.xh[i & 1][sd];
      pa.oix[sd] = i == last ? s.ix[sd] : s.xix[i & 1][sd];
    }
    count_launch();
    if (i == 0) {
      if ((err = ensure_dyn_smem<k_part_pass<true>>(psmem)) != cudaSuccess) return err;
      k_part_pass<true><<<(unsigned)((pa.n + kPassTile - 1) / kPassTile), kPassThreads, psmem, st>>>(pa);
    } else {
      pa.P = (uint32_t)pl.children[i - 1];
      pa.icap = pl.cap[i - 1];
      pa.icnt = s.cnt + pl.cnt_off[i - 1];
      pa.tiles_per_parent = (uint32_t)((pa.icap + kPassTile - 1) / kPassTile);
      for (int sd = 0; sd < 2; sd++) {
        pa.ih[sd] = s.xh[(i - 1) & 1][sd];
        pa.iix[sd] = s.xix[(i - 1) & 1][sd];
      }
      if ((err = ensure_dyn_smem<k_part_pass<false>>(psmem)) != cudaSuccess) return err;
      k_part_pass<false><<<(unsigned)(2 * pa.P * pa.tiles_per_parent), kPassThreads, psmem, st>>>(pa);
    }
    if ((err = cudaGetLastError()) != cudaSuccess) return err;
  }
  if ((err = scan_apply<uint32_t>(BucketCountIn{s.bcnt, (uint32_t)s.side_cap}, (int64_t)B, s.scan,
                                  BucketOffOut{s.roff, (int64_t)B}, st)) !=
      cudaSuccess)
    return err;
  MatchArgs ma;
  ma.a = a;
  ma.h[0] = s.h[0];
  ma.h[1] = s.h[1];
  ma.ix[0] = s.ix[0];
  ma.ix[1] = s.ix[1];
  ma.cnt = s.bcnt;
  ma.roff = s.roff;
  ma.sflag[0] = s.sflag[0];
  ma.sflag[1] = s.sflag[1];
  ma.overflow = s.overflow;
  ma.B = B;
  if (ordered) return launch_bucket_match<true, 256, 128, 6>(ma, B, st);
#if MM_UNORD_POP
  {
    constexpr int kA = MM_UNORD_AVG, kT = kA == 512 ? 256 : 128, kB = kA == 512 ? 3 : 6;
    constexpr auto kern = k_bucket_pop<kA, kT, kB>;
    const size_t smem = sizeof(PopSmem<4 * kA, 8 * kA, kT>);
    if ((err = ensure_dyn_smem<kern>(smem)) != cudaSuccess) return err;
    count_launch();
    kern<<<persistent_grid<kern>(kT, smem, B), kT, smem, st>>>(ma);
    return cudaGetLastError();
  }
#endif
  return launch_bucket_match<false, 512, 256, 3>(ma, B, st);
}

// Partly matched side: the bucket slots' matched bytes scattered to snapshot
// order, so that the compaction keeps the residual queue in posting / arrival
// order (run_compact).
__global__ void k_slot_flags(const uint32_t* cnt, const uint32_t* ix, const uint8_t* sflag, int64_t nslots,
                             int64_t side_cap, uint8_t* flag) {
  for (int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; s < nslots; s += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = s / side_cap;
    if ((uint32_t)(s - b * side_cap) < cnt[b]) flag[ix[s]] = sflag[s];
  }
}
cudaError_t run_slot_flags(const BucketScratch& s, int side, uint8_t* flag, cudaStream_t st) {
  const int64_t nslots = (int64_t)s.B * s.side_cap;
  int64_t g = (nslots + 255) / 256;
  if (g > 148 * 16) g = 148 * 16;
  count_launch();
  k_slot_flags<<<(unsigned)g, 256, 0, st>>>(s.bcnt + (side ? s.B : 0), s.ix[side], s.sflag[side], nslots, s.side_cap,
                                            flag);
  return cudaGetLastError();
}

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
