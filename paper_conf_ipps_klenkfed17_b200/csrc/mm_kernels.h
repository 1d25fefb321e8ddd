// mm_kernels.h -- argument blocks and launchers of the matching kernels.
#pragma once

#include "mm_internal.cuh"

namespace mm {

struct MpiArgs {
  Side R, M;
  int n_ep;      // endpoints [ep0, n_ep) are matched by this launch
  int ep0 = 0;
  int64_t msg_slots;        // shared-memory message slots per warp (>= msg cap, multiple of 64)
  int64_t warp_smem_words;  // 8-byte words of shared memory per warp
  int64_t* out_rc;
  int64_t* out_mc;
  int64_t out_cap;
  const int64_t* out_off;
  uint64_t* q_rh_w;
  int64_t* q_rc_w;
  int32_t* rres_w;
  uint64_t* q_mh_w;
  int64_t* q_mc_w;
  int32_t* mres_w;
  unsigned long long* n_matched;
  uint32_t* err;
};

// Key-FIFO engine workspace (byte offsets inside one CTA's workspace).
constexpr int64_t kFifoSmemMax = 100 * 1024;
struct FifoLayout {
  int64_t whdr, keyhdr, table, key_cnt, key_start, key_rcnt, key_rstart, key_c, msg_key, by_key,
      wlog, recv_key, recv_e, rby_key, recv_res, wl, matched, pcnt, gnext, gfirst, gwc, w_grp, mcap;
  int64_t total;
  uint32_t H;
  uint32_t wcap;
  bool in_smem;
  // global-workspace variant: the arrays the serial parts chase (by_key,
  // rby_key, wl, recv_key) staged in the CTA's shared memory when they fit
  int64_t stage_bytes = 0, st_by_key = 0, st_rby_key = 0, st_wl = 0, st_recv_key = 0;
  int64_t st_wlog = -1;  // staged wildcard-claim log (P7..P8) when it fits, else -1
  int64_t lead_runw = -1;  // global workspace: run positions of the data-parallel leading runs, else -1
  int cluster = 1;         // CTAs per deep endpoint (thread-block cluster), 1 = one CTA
};
FifoLayout fifo_layout(int64_t rcap, int64_t mcap, int n_ep);
int fifo_grid(const FifoLayout& L, int n_ep);
cudaError_t launch_mpi_fifo(const MpiArgs& a, const FifoLayout& L, uint8_t* gws, cudaStream_t st);

cudaError_t launch_out_offsets(const Side& R, int n_ep, int64_t* out_off, int64_t out_cap, uint32_t* err,
                               unsigned long long* n_matched, cudaStream_t st);
cudaError_t launch_mpi_matrix(const MpiArgs& a, cudaStream_t st);

// Append the pending elements of every endpoint to its queue (used when a
// second post/push arrives before a match).
cudaError_t launch_materialize(const Side& S, int n_ep, uint64_t* q_h, int64_t* q_c, int32_t* q_len, uint32_t* err,
                               cudaStream_t st);

// ------------------------------------------------- no-wildcard levels (n_ep = 1)
struct FlatArgs {
  Side R, M;
  int64_t nr, nm;  // exact snapshot sizes (host-known)
  unsigned long long* n_matched;
  int64_t* out_rc;
  int64_t* out_mc;
  uint8_t* rflag;  // 1 = receive matched
  uint8_t* mflag;  // 1 = message matched
};

struct SnapInfo {
  unsigned long long diff;  // OR over all snapshot headers of (hdr ^ ref)
  unsigned long long ref;
  int32_t rres, mres;
};
cudaError_t launch_snapshot_info(const Side& R, const Side& M, int64_t bound, SnapInfo* info, bool want_diff,
                                 cudaStream_t st);

// Ordered level: sort-and-rank pairing (row A4).
struct SortScratch {
  uint64_t* key[2];
  uint32_t* val[2];
  uint32_t* rid;
  uint32_t* run_start;
  uint32_t* run_rc;
  uint32_t* part;  // partition scratch
  unsigned long long* scan;
};
cudaError_t run_sort_rank(const FlatArgs& a, uint64_t ref, uint64_t diff, const SortScratch& s, cudaStream_t st);

// Unordered level: lock-free open-addressing hash table (row A5).
struct HashScratch {
  uint32_t* owner;  // [T] receive index owning the slot (EMPTY = 0xFFFFFFFF)
  uint32_t* rcnt;   // [T] receives with the slot's tuple
  uint32_t* mcnt;   // [T] messages that probed the slot
  unsigned long long* tkey;  // [T] ticket table keys (slot << 32 | ticket)
  uint32_t* tval;            // [T] receive index of a ticket
  int64_t T;                 // power of two
};
cudaError_t run_hash(const FlatArgs& a, const HashScratch& h, cudaStream_t st);

// Gate of the device-decided tail of a bucketed batch (one thread): sets the
// graph's conditional handles (fallback / partly matched receives / partly
// matched messages), empties the residual queue of a fully matched side,
// counts fallbacks and, without one, writes the counts {nr, pairs} (engine
// and, if given, caller).
cudaError_t launch_flat_gate(const uint32_t* over, const unsigned long long* n_matched, int64_t nr, int64_t nm,
                             cudaGraphConditionalHandle hfb, cudaGraphConditionalHandle hr,
                             cudaGraphConditionalHandle hm, cudaGraphConditionalHandle hany, int32_t* len_r,
                             int32_t* len_m, unsigned long long* fallbacks, int64_t* counts, int64_t* user_counts,
                             cudaStream_t st);

// Both no-wildcard levels, hash-bucketed (k_bucket.cu): one-pass partition
// into fixed-capacity bucket regions + one CTA per bucket.  Sets *overflow if
// a bucket does not fit (the caller then falls back to run_sort_rank /
// run_hash).
constexpr int kMaxPasses = 4;
struct PartPlan {                 // partition passes for a side of n_side elements (k_bucket.cu)
  int nb, passes;
  int bits[kMaxPasses], shift[kMaxPasses];
  int64_t children[kMaxPasses];   // regions per side after pass i
  int64_t cap[kMaxPasses];        // slots per region after pass i
  int64_t slots[kMaxPasses];      // children x cap
  int64_t cnt_off[kMaxPasses];    // offset of pass i's counts [2][children] in the count array
  int64_t cnt_total;
  int64_t scratch_slots[2];       // intermediate levels alternate between two buffers
};
PartPlan part_plan(int64_t n_side, int avg);
PartPlan part_plan_alloc(int64_t n_side, int avg);  // the largest any batch up to n_side needs
struct BucketScratch {
  uint64_t* h[2];      // final bucket regions (plan.slots[last]): headers (receives, messages)
  uint32_t* ix[2];     // ... snapshot indices
  uint8_t* sflag[2];   // ... matched byte per slot
  uint64_t* xh[2][2];  // intermediate regions [buffer][side]
  uint32_t* xix[2][2];
  uint32_t* cnt;       // every pass's region counts (plan.cnt_total), then the overflow flag
  uint32_t* roff;      // [B + 1] output offsets of the buckets
  uint32_t* scan;      // scan scratch (scan_scratch_elems(B))
  uint32_t* overflow;  // = cnt + plan.cnt_total (set by run_bucketed)
  int64_t rres, mres;
  PartPlan plan;       // set by run_bucketed
  int64_t side_cap;    // region slots per side and bucket (set by run_bucketed)
  const uint32_t* bcnt;  // final counts [2][B] (set by run_bucketed)
  uint32_t B;
};
int bucket_avg(bool ordered);  // bucket geometry: average elements per side and bucket
int bucket_bits_for(int64_t n_side, int avg);
int64_t bucket_count(int64_t n_side, int avg);
cudaError_t run_bucketed(const FlatArgs& a, bool ordered, BucketScratch& s, cudaStream_t st);
// snapshot-order matched flags of one side from the bucket slots (partly matched sides)
cudaError_t run_slot_flags(const BucketScratch& s, int side, uint8_t* flag, cudaStream_t st);

// Compaction of the no-wildcard queues into the other ping-pong buffer.
cudaError_t run_compact(const Side& S, int64_t resid, int64_t n, const uint8_t* matched, uint64_t* q_h, int64_t* q_c,
                        int32_t* q_len, uint32_t* scan, cudaStream_t st);

// mm_route
cudaError_t run_route(const uint64_t* a, const int64_t* b, int64_t n, int world, int by, int64_t cookie_base, uint64_t* out_a,
                      int64_t* out_b, int64_t* counts, uint32_t* part, cudaStream_t st);

// counts[] = {n_out, n_matched} from device state
cudaError_t launch_reset(int32_t* rlen, int32_t* mlen, int n_ep, uint32_t* err, unsigned long long* n_matched,
                         cudaStream_t st);
cudaError_t launch_finalize(const int64_t* n_out_src, int64_t n_out_host, const unsigned long long* n_matched,
                            int64_t* counts, int64_t* user_counts, cudaStream_t st);

}  // namespace mm
