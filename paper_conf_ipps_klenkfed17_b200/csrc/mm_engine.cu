// mm_engine.cu -- the C-ABI of include/mm.h (host side).
//
// Owns the per-endpoint queues in HBM, stages host buffers, and sequences the
// kernels of k_mpi.cu / k_flat.cu on the engine's stream.  No matching
// arithmetic happens on the host.
#include <nvtx3/nvToolsExt.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <new>

#include "mm_kernels.h"

using namespace mm;

namespace mm {
long long& launch_count() {
  static long long n = 0;
  return n;
}
}  // namespace mm

namespace {

// Ring of CUDA event pairs bracketing the dominant kernel region of each
// mm_match_batch; resolved lazily so timing never blocks the launch stream.
struct Timer {
  static constexpr int kRing = 64;
  cudaEvent_t a[kRing] = {}, b[kRing] = {};
  int head = 0, count = 0;  // pending pairs: [head - count, head)
  bool ok = false;
  long long ns = 0, runs = 0;
  void init() {
    ok = true;
    for (int i = 0; i < kRing; i++)
      if (cudaEventCreate(&a[i]) != cudaSuccess || cudaEventCreate(&b[i]) != cudaSuccess) ok = false;
    if (!ok) cudaGetLastError();
  }
  void destroy() {
    for (int i = 0; i < kRing; i++) {
      if (a[i]) cudaEventDestroy(a[i]);
      if (b[i]) cudaEventDestroy(b[i]);
      a[i] = b[i] = nullptr;
    }
  }
  void resolve_one() {
    int i = (head - count + kRing) % kRing;
    float ms = 0.f;
    if (cudaEventSynchronize(b[i]) == cudaSuccess && cudaEventElapsedTime(&ms, a[i], b[i]) == cudaSuccess) {
      ns += (long long)(ms * 1e6);
      runs++;
    } else {
      cudaGetLastError();
    }
    count--;
  }
  void resolve_all() {
    while (count > 0) resolve_one();
  }
  // The region is also an NVTX push/pop range "mm_region" (free without a
  // tool attached): `ncu --nvtx --nvtx-include "mm_region]"` captures exactly
  // the launches the CUDA-event time covers (bench.py roofline.traffic).
  void begin(cudaStream_t st) {
    nvtxRangePushA("mm_region");
    if (!ok) return;
    if (count == kRing) resolve_one();
    cudaEventRecord(a[head], st);
  }
  void end(cudaStream_t st) {
    nvtxRangePop();
    if (!ok) return;
    cudaEventRecord(b[head], st);
    head = (head + 1) % kRing;
    count++;
  }
};

struct DBuf {
  void* p = nullptr;
  size_t bytes = 0;
};

cudaError_t ensure(DBuf& b, size_t bytes) {
  if (bytes == 0) bytes = 16;
  if (b.bytes >= bytes) return cudaSuccess;
  if (b.p) cudaFree(b.p);
  b.p = nullptr;
  b.bytes = 0;
  cudaError_t err = cudaMalloc(&b.p, bytes);
  if (err == cudaSuccess) b.bytes = bytes;
  return err;
}

void release(DBuf& b) {
  if (b.p) cudaFree(b.p);
  b.p = nullptr;
  b.bytes = 0;
}

// Device address of page-locked (mapped) host memory, or nullptr for
// pageable host memory and device memory.
static void* mapped_host_ptr(const void* p) {
  if (!p) return nullptr;
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return at.type == cudaMemoryTypeHost ? at.devicePointer : nullptr;
}

bool is_device_ptr(const void* p) {
  if (!p) return false;
  cudaPointerAttributes at;
  cudaError_t err = cudaPointerGetAttributes(&at, p);
  if (err != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

int64_t next_pow2(int64_t x) {
  int64_t p = 1;
  while (p < x) p <<= 1;
  return p;
}

struct Pending {
  const uint64_t* hdr = nullptr;
  const int64_t* cookie = nullptr;
  const int64_t* off = nullptr;
  int64_t n = 0;
  int64_t seq0 = 0;
  bool active = false;
  int chunks = 0;  // > 0: host input staged in `chunks` endpoint ranges on the copy stream (Queue::ev)
  bool issued = false;  // the chunk copies are submitted (deferred so both queues' chunks interleave)
  const uint64_t* h_hdr = nullptr;  // the caller's host buffers (valid until mm_match_batch returns)
  const int64_t* h_cookie = nullptr;
  const int64_t* h_off = nullptr;
};

// Host-buffer pipeline (MPI level): endpoint range k of C is [k*n_ep/C, (k+1)*n_ep/C).
constexpr int kMaxChunks = 32;

struct Queue {
  DBuf hdr[2], cookie[2], len[2];  // ping-pong (the MPI level compacts in place and uses [0] only)
  DBuf st_hdr, st_cookie, st_off;   // staging for host inputs
  Pending pend;
  cudaEvent_t ev[kMaxChunks] = {};  // chunk k of the pending host input is on the device
  int64_t seq = 0;
  int cur = 0;
  int64_t resid_host = 0;  // residual count (single-endpoint levels): exact if resid_exact, else an upper bound
  bool resid_exact = true;
};

}  // namespace

#ifndef MM_TAIL_SIDE
#define MM_TAIL_SIDE 1  // A/B: the tail graph launched on the side stream
#endif
#ifndef MM_FLAT_TAIL
#define MM_FLAT_TAIL 1  // device-decided tail of bucketed no-wildcard batches (0: host read-back)
#endif

struct mm_engine {
  int sem = 0;
  int n_ep = 1;
  int64_t rcap = 0, mcap = 0;
  cudaStream_t st = nullptr;
  int dev = 0;
  Queue rq, mq;
  DBuf out_off, counts_dev, nmatched, err, info;
  DBuf out_rc_stage, out_mc_stage;
  // MPI
  int64_t msg_slots = 0, warp_words = 0;
  int mpi_kernel = MM_MPI_KERNEL_FIFO;
  bool mpi_resid_empty = true;  // no residual receive anywhere (after create / reset, before a match)
  FifoLayout fifo{};
  DBuf fifo_ws;
  // single-endpoint levels
  DBuf rflag, mflag, scan;
  DBuf skey[2], sval[2], rid, run_start, run_rc, part;
  DBuf owner, rcnt, mcnt, tkey, tval;
  int64_t T = 0;
  DBuf bh[2], bix[2], bsflag[2], bxh[2][2], bxix[2][2], bcnt, broff, bscan;  // bucket regions (k_bucket.cu)
  int flat_kernel = MM_FLAT_KERNEL_BUCKETED;
  long long bucket_fallbacks = 0;
  // Device-decided tail of bucketed no-wildcard batches (flat_tail): a CUDA
  // graph whose conditional nodes run the global fallback and the
  // compactions as the overflow flag and the pair count decide on the
  // device, so the batch needs no host read-back.  Instantiated graphs are
  // cached by everything their launches capture (TailKey).
  struct TailKey {
    FlatArgs a;
    const void* ptr[26];
    int64_t val[8];
  };
  struct TailGraph {
    TailKey key;
    cudaGraphExec_t exec = nullptr;
    long long stamp = 0;
  };
  static constexpr int kTailCache = 4;
  TailGraph tails[kTailCache];
  long long tail_clock = 0;
  cudaStream_t gs = nullptr;  // capture stream
  DBuf fb_dev;                // fallbacks taken by device-decided tails
  int tail_mode = 1;          // MM_FLAT_TAIL A/B: 0 = host read-back of the overflow flag and the pair count
  bool nm_zero = false;       // the pair counter is zero (mm_reset's kernel cleared it, no batch since)
  Timer timer;
  long long launches = 0;
  // host-buffer pipeline: H2D copies on cs, D2H copies on ds, chunk kernels on st
  cudaStream_t cs = nullptr, ds = nullptr;
  cudaEvent_t ev_st = nullptr, ev_k[kMaxChunks] = {};
  int64_t* h_off = nullptr;  // pinned copy of out_off (n_ep + 1)
  // pinned landing zone of the small per-batch read-backs (truly asynchronous
  // copies, no staging through pageable memory)
  struct Small {
    SnapInfo info;
    unsigned long long matched;
    unsigned long long tail_matched;  // pair count of the last device-decided tail (read back asynchronously)
    uint32_t over;
  }* h_small = nullptr;
  // after a device-decided tail with device buffers the residual sizes are
  // exact again (resid_host = snapshot - pairs) once ev_nm has completed:
  // the next batch then fetches the pair count on the side stream
  cudaEvent_t ev_nm = nullptr;
  bool nm_pending = false;
  cudaEvent_t ev_tail[2] = {nullptr, nullptr};  // orders the tail graph's side-stream launch
  int pipeline = 0;          // MM_OPT_PIPELINE_CHUNKS (0 = auto)
  int host_out = MM_HOST_OUT_STAGED;  // MM_OPT_HOST_OUT
  // copies out of the caller's host input buffers still in flight: recorded
  // after they are issued (on st by post, on cs by issue_chunks) and waited
  // for before mm_match_batch / mm_reset return, so that the caller may
  // refill those buffers (page-locked ones included) once the call returns
  cudaEvent_t ev_in_st = nullptr, ev_in_cs = nullptr;
  bool in_st = false, in_cs = false;
};

// Wait until every copy out of the caller's host input buffers has executed.
static cudaError_t release_host_inputs(mm_engine* e) {
  cudaError_t r = cudaSuccess;
  if (e->in_st) r = cudaEventSynchronize(e->ev_in_st);
  if (r == cudaSuccess && e->in_cs) r = cudaEventSynchronize(e->ev_in_cs);
  e->in_st = e->in_cs = false;
  return r;
}

// Range k of C covers endpoints [chunk_ep(k), chunk_ep(k + 1)).  Ranges grow
// linearly towards the middle (weights min(j + 1, C - j)): the first range's
// copy-in and the last range's copy-out are the only transfers nothing
// overlaps, so they are the smallest.
#ifndef MM_PIPE_RAMP
#define MM_PIPE_RAMP 1  // A/B: 0 = equal ranges (e2e 2.07-2.10 vs 1.93-1.97 ms at 4-6 ranges)
#endif
static int64_t chunk_weight_sum(int k, int C) {
  int64_t s = 0;
  for (int j = 0; j < k; j++) s += MM_PIPE_RAMP ? ((j + 1 < C - j) ? j + 1 : C - j) : 1;
  return s;
}
static int64_t chunk_ep(const mm_engine* e, int k, int C) {
  return (int64_t)e->n_ep * chunk_weight_sum(k, C) / chunk_weight_sum(C, C);
}

// Number of endpoint ranges the host-buffer pipeline uses (1 = no pipeline).
static int pipeline_chunks(const mm_engine* e) {
  if (e->sem != MM_SEM_MPI || e->n_ep < 2) return 1;
  int C = e->pipeline;
  if (C == 0) C = e->n_ep >= 1024 ? 6 : (e->n_ep >= 256 ? 4 : 1);
  return C < e->n_ep ? C : e->n_ep;
}

// Attributes the library's kernel launches during one API call to an engine.
struct LaunchScope {
  mm_engine* e;
  long long start;
  explicit LaunchScope(mm_engine* en) : e(en), start(mm::launch_count()) {}
  ~LaunchScope() {
    if (e) e->launches += mm::launch_count() - start;
  }
};

// MM_DEBUG=1 in the environment: every failing CUDA call is reported on
// stderr (file:line and the CUDA error) before MM_ERR_CUDA is returned.
static int ck_fail(cudaError_t e, int line) {
  static const bool dbg = getenv("MM_DEBUG") != nullptr;
  if (dbg) fprintf(stderr, "mm_engine.cu:%d: %s\n", line, cudaGetErrorString(e));
  return MM_ERR_CUDA;
}
#define CK(x)                                               \
  do {                                                      \
    cudaError_t _e = (x);                                   \
    if (_e != cudaSuccess) return ck_fail(_e, __LINE__);    \
  } while (0)

static Side make_side(mm_engine* e, Queue& q, int64_t cap) {
  Side s;
  s.q_hdr = (const uint64_t*)q.hdr[q.cur].p;
  s.q_cookie = (const int64_t*)q.cookie[q.cur].p;
  s.q_len = (const int32_t*)q.len[q.cur].p;
  s.p_hdr = q.pend.active ? q.pend.hdr : nullptr;
  s.p_cookie = q.pend.active ? q.pend.cookie : nullptr;
  s.p_off = q.pend.active ? q.pend.off : nullptr;
  s.p_n = q.pend.active ? q.pend.n : 0;
  s.p_seq0 = q.pend.seq0;
  s.cap = cap;
  (void)e;
  return s;
}

static int alloc_queue(mm_engine* e, Queue& q, int64_t cap, bool pingpong) {
  const int64_t slots = (int64_t)e->n_ep * cap;
  for (int b = 0; b < (pingpong ? 2 : 1); b++) {
    CK(ensure(q.hdr[b], slots * 8));
    CK(ensure(q.cookie[b], slots * 8));
    CK(ensure(q.len[b], (size_t)e->n_ep * 4));
    CK(cudaMemsetAsync(q.len[b].p, 0, (size_t)e->n_ep * 4, e->st));
  }
  return MM_OK;
}

extern "C" {

const char* mm_strerror(int code) {
  switch (code) {
    case MM_OK: return "ok";
    case MM_ERR_ARG: return "invalid argument";
    case MM_ERR_CUDA: return "CUDA runtime error";
    case MM_ERR_CAPACITY: return "queue or output capacity exceeded";
    case MM_ERR_NOMEM: return "out of memory";
    case MM_ERR_STATE: return "invalid state";
    default: return "unknown error";
  }
}

const char* mm_version(void) { return "mm 0.1.0 sm_100a"; }

int mm_destroy(mm_engine* e) {
  if (!e) return MM_OK;
  cudaStreamSynchronize(e->st);
  if (e->cs) cudaStreamSynchronize(e->cs);
  if (e->ds) cudaStreamSynchronize(e->ds);
  e->timer.destroy();
  Queue* qs[2] = {&e->rq, &e->mq};
  for (int k = 0; k < kMaxChunks; k++) {
    if (e->ev_k[k]) cudaEventDestroy(e->ev_k[k]);
    for (Queue* q : qs)
      if (q->ev[k]) cudaEventDestroy(q->ev[k]);
  }
  if (e->ev_st) cudaEventDestroy(e->ev_st);
  if (e->ev_in_st) cudaEventDestroy(e->ev_in_st);
  if (e->ev_in_cs) cudaEventDestroy(e->ev_in_cs);
  for (auto& t : e->tails)
    if (t.exec) cudaGraphExecDestroy(t.exec);
  if (e->gs) cudaStreamDestroy(e->gs);
  if (e->ev_nm) cudaEventDestroy(e->ev_nm);
  for (cudaEvent_t ev : e->ev_tail)
    if (ev) cudaEventDestroy(ev);
  if (e->cs) cudaStreamDestroy(e->cs);
  if (e->ds) cudaStreamDestroy(e->ds);
  if (e->h_off) cudaFreeHost(e->h_off);
  if (e->h_small) cudaFreeHost(e->h_small);
  for (Queue* q : qs) {
    for (int b = 0; b < 2; b++) {
      release(q->hdr[b]);
      release(q->cookie[b]);
      release(q->len[b]);
    }
    release(q->st_hdr);
    release(q->st_cookie);
    release(q->st_off);
  }
  DBuf* bufs[] = {&e->out_off, &e->counts_dev, &e->nmatched, &e->err, &e->info, &e->out_rc_stage,
                  &e->out_mc_stage, &e->rflag, &e->mflag, &e->scan, &e->skey[0], &e->skey[1],
                  &e->sval[0], &e->sval[1], &e->rid, &e->run_start, &e->run_rc, &e->part,
                  &e->owner, &e->rcnt, &e->mcnt, &e->tkey, &e->tval, &e->fifo_ws,
                  &e->bh[0], &e->bh[1], &e->bix[0], &e->bix[1], &e->bsflag[0], &e->bsflag[1], &e->bcnt,
                  &e->broff, &e->bscan, &e->bxh[0][0], &e->bxh[0][1], &e->bxh[1][0], &e->bxh[1][1],
                  &e->bxix[0][0], &e->bxix[0][1], &e->bxix[1][0], &e->bxix[1][1], &e->fb_dev};
  for (DBuf* b : bufs) release(*b);
  delete e;
  return MM_OK;
}

int mm_create(mm_engine** out, int32_t semantics, int32_t n_endpoints, int64_t recv_capacity, int64_t msg_capacity,
              void* stream) {
  if (!out) return MM_ERR_ARG;
  *out = nullptr;
  if (semantics < MM_SEM_MPI || semantics > MM_SEM_NOWILD_UNORDERED) return MM_ERR_ARG;
  if (n_endpoints < 1 || recv_capacity < 1 || msg_capacity < 1) return MM_ERR_ARG;
  if (semantics != MM_SEM_MPI && n_endpoints != 1) return MM_ERR_ARG;
  if (semantics == MM_SEM_MPI && (msg_capacity > MM_MPI_MAX_MSGS || recv_capacity > MM_MPI_MAX_RECVS))
    return MM_ERR_ARG;
  if (semantics != MM_SEM_MPI && recv_capacity + msg_capacity >= (int64_t)1 << 31) return MM_ERR_ARG;
  mm_engine* e = new (std::nothrow) mm_engine();
  if (!e) return MM_ERR_NOMEM;
  e->sem = semantics;
  e->n_ep = n_endpoints;
  e->rcap = recv_capacity + (recv_capacity & 1);  // even stride keeps 16-byte alignment
  e->mcap = msg_capacity + (msg_capacity & 1);
  e->st = (cudaStream_t)stream;
  if (cudaGetDevice(&e->dev) != cudaSuccess) {
    cudaGetLastError();
    delete e;
    return MM_ERR_CUDA;
  }
  int rc = MM_OK;
  const bool pp = semantics != MM_SEM_MPI;
  if (cudaMallocHost(&e->h_small, sizeof(*e->h_small)) != cudaSuccess) {
    cudaGetLastError();
    delete e;
    return MM_ERR_NOMEM;
  }
  if ((rc = alloc_queue(e, e->rq, e->rcap, pp)) != MM_OK || (rc = alloc_queue(e, e->mq, e->mcap, pp)) != MM_OK) {
    mm_destroy(e);
    return rc == MM_ERR_CUDA ? MM_ERR_NOMEM : rc;
  }
  bool ok = ensure(e->out_off, (size_t)(n_endpoints + 1) * 8) == cudaSuccess &&
            ensure(e->counts_dev, 16) == cudaSuccess && ensure(e->nmatched, 8) == cudaSuccess &&
            ensure(e->err, 4) == cudaSuccess && ensure(e->info, sizeof(SnapInfo)) == cudaSuccess;
  // (every level: host inputs are copied out of the caller's buffers)
  ok = ok && cudaEventCreateWithFlags(&e->ev_in_st, cudaEventDisableTiming) == cudaSuccess &&
       cudaEventCreateWithFlags(&e->ev_in_cs, cudaEventDisableTiming) == cudaSuccess;
  if (ok && semantics != MM_SEM_MPI) {
    ok = cudaStreamCreateWithFlags(&e->gs, cudaStreamNonBlocking) == cudaSuccess &&
         cudaEventCreateWithFlags(&e->ev_nm, cudaEventDisableTiming) == cudaSuccess &&
         cudaEventCreateWithFlags(&e->ev_tail[0], cudaEventDisableTiming) == cudaSuccess &&
         cudaEventCreateWithFlags(&e->ev_tail[1], cudaEventDisableTiming) == cudaSuccess &&
         ensure(e->fb_dev, 8) == cudaSuccess && cudaMemset(e->fb_dev.p, 0, 8) == cudaSuccess;
    e->tail_mode = MM_FLAT_TAIL;
  }
  if (ok && semantics == MM_SEM_MPI) {
    ok = cudaStreamCreateWithFlags(&e->cs, cudaStreamNonBlocking) == cudaSuccess &&
         cudaStreamCreateWithFlags(&e->ds, cudaStreamNonBlocking) == cudaSuccess &&
         cudaEventCreateWithFlags(&e->ev_st, cudaEventDisableTiming) == cudaSuccess &&
         cudaMallocHost(&e->h_off, (size_t)(n_endpoints + 1) * 8) == cudaSuccess;
    for (int k = 0; ok && k < kMaxChunks; k++)
      ok = cudaEventCreateWithFlags(&e->ev_k[k], cudaEventDisableTiming) == cudaSuccess &&
           cudaEventCreateWithFlags(&e->rq.ev[k], cudaEventDisableTiming) == cudaSuccess &&
           cudaEventCreateWithFlags(&e->mq.ev[k], cudaEventDisableTiming) == cudaSuccess;
  }
  if (ok && semantics == MM_SEM_MPI) {
    e->msg_slots = (e->mcap + 63) / 64 * 64;
    e->warp_words = (e->msg_slots + e->msg_slots / 64 + 3) / 4 * 4;  // headers + availability bits, 32 B aligned
    e->fifo = fifo_layout(e->rcap, e->mcap, n_endpoints);
    if (!e->fifo.in_smem)
      ok = ensure(e->fifo_ws, (size_t)fifo_grid(e->fifo, n_endpoints) * (size_t)e->fifo.total) == cudaSuccess;
  }
  if (ok && semantics != MM_SEM_MPI) {
    const int64_t n = e->rcap + e->mcap;
    ok = ensure(e->rflag, e->rcap) == cudaSuccess && ensure(e->mflag, e->mcap) == cudaSuccess &&
         ensure(e->scan, (size_t)scan_scratch_elems(n) * 8) == cudaSuccess;
    // bucket regions sized for the larger side (k_bucket.cu)
    const int64_t side = e->rcap > e->mcap ? e->rcap : e->mcap;
    const int avg = bucket_avg(semantics == MM_SEM_NOWILD_ORDERED);
    const PartPlan pl = part_plan_alloc(side, avg);
    const int64_t nbk = bucket_count(side, avg), slots = nbk * pl.cap[pl.passes - 1];
    for (int b = 0; ok && b < 2; b++) {
      ok = ensure(e->bh[b], (size_t)slots * 8) == cudaSuccess && ensure(e->bix[b], (size_t)slots * 4) == cudaSuccess &&
           ensure(e->bsflag[b], (size_t)slots) == cudaSuccess;
      for (int x = 0; ok && x < 2; x++)
        if (pl.scratch_slots[x] > 0)
          ok = ensure(e->bxh[x][b], (size_t)pl.scratch_slots[x] * 8) == cudaSuccess &&
               ensure(e->bxix[x][b], (size_t)pl.scratch_slots[x] * 4) == cudaSuccess;
    }
    ok = ok && ensure(e->bcnt, (size_t)(pl.cnt_total + 1) * 4) == cudaSuccess &&
         ensure(e->broff, (size_t)(nbk + 1) * 4) == cudaSuccess &&
         ensure(e->bscan, (size_t)scan_scratch_elems(nbk) * 4) == cudaSuccess;
    if (ok && semantics == MM_SEM_NOWILD_ORDERED) {
      ok = ensure(e->skey[0], n * 8) == cudaSuccess && ensure(e->skey[1], n * 8) == cudaSuccess &&
           ensure(e->sval[0], n * 4) == cudaSuccess && ensure(e->sval[1], n * 4) == cudaSuccess &&
           ensure(e->rid, n * 4) == cudaSuccess && ensure(e->run_start, (n + 2) * 4) == cudaSuccess &&
           ensure(e->run_rc, (n + 2) * 4) == cudaSuccess &&
           ensure(e->part, (size_t)partition_scratch_elems(n) * 4) == cudaSuccess;
    }
    if (ok && semantics == MM_SEM_NOWILD_UNORDERED) {
      e->T = next_pow2(2 * e->rcap < 1024 ? 1024 : 2 * e->rcap);
      ok = ensure(e->owner, e->T * 4) == cudaSuccess && ensure(e->rcnt, e->T * 4) == cudaSuccess &&
           ensure(e->mcnt, e->T * 4) == cudaSuccess && ensure(e->tkey, e->T * 8) == cudaSuccess &&
           ensure(e->tval, e->T * 4) == cudaSuccess;
    }
  }
  if (!ok) {
    cudaGetLastError();
    mm_destroy(e);
    return MM_ERR_NOMEM;
  }
  if (cudaMemsetAsync(e->err.p, 0, 4, e->st) != cudaSuccess || cudaMemsetAsync(e->nmatched.p, 0, 8, e->st) != cudaSuccess) {
    mm_destroy(e);
    return MM_ERR_CUDA;
  }
  e->timer.init();
  *out = e;
  return MM_OK;
}

// Submit the chunk copies of the deferred host inputs of queues qs[0..nq),
// range by range (range k of every queue before range k + 1 of any).
static int issue_chunks(mm_engine* e, Queue** qs, int nq) {
  bool any = false;
  for (int i = 0; i < nq; i++) any |= qs[i]->pend.active && qs[i]->pend.chunks > 0 && !qs[i]->pend.issued;
  if (!any) return MM_OK;
  CK(cudaEventRecord(e->ev_st, e->st));  // the staging buffers are free once earlier work on st is done
  CK(cudaStreamWaitEvent(e->cs, e->ev_st, 0));
  for (int k = 0; k < kMaxChunks; k++)
    for (int i = 0; i < nq; i++) {
      Pending& p = qs[i]->pend;
      if (!p.active || p.chunks <= k || p.issued) continue;
      const int64_t a = p.h_off[chunk_ep(e, k, p.chunks)], b = p.h_off[chunk_ep(e, k + 1, p.chunks)];
      if (b > a) {
        CK(cudaMemcpyAsync((uint64_t*)p.hdr + a, p.h_hdr + a, (size_t)(b - a) * 8, cudaMemcpyHostToDevice, e->cs));
        if (p.h_cookie)
          CK(cudaMemcpyAsync((int64_t*)p.cookie + a, p.h_cookie + a, (size_t)(b - a) * 8, cudaMemcpyHostToDevice,
                             e->cs));
      }
      CK(cudaEventRecord(qs[i]->ev[k], e->cs));
    }
  for (int i = 0; i < nq; i++)
    if (qs[i]->pend.active && qs[i]->pend.chunks > 0) qs[i]->pend.issued = true;
  CK(cudaEventRecord(e->ev_in_cs, e->cs));
  e->in_cs = true;
  return MM_OK;
}

// Order the engine stream after every chunk copy of q's pending host input.
static int join_pending(mm_engine* e, Queue& q) {
  if (!q.pend.active || q.pend.chunks == 0) return MM_OK;
  Queue* qs[1] = {&q};
  int rc = issue_chunks(e, qs, 1);
  if (rc != MM_OK) return rc;
  CK(cudaStreamWaitEvent(e->st, q.ev[q.pend.chunks - 1], 0));
  return MM_OK;
}

static int materialize(mm_engine* e, Queue& q, int64_t cap) {
  if (!q.pend.active) return MM_OK;
  e->mpi_resid_empty = false;
  int jr = join_pending(e, q);
  if (jr != MM_OK) return jr;
  Side s = make_side(e, q, cap);
  CK(launch_materialize(s, e->n_ep, (uint64_t*)q.hdr[q.cur].p, (int64_t*)q.cookie[q.cur].p, (int32_t*)q.len[q.cur].p,
                        (uint32_t*)e->err.p, e->st));
  q.resid_host += q.pend.n;
  if (q.resid_host > cap) {
    q.resid_host = cap;
    q.resid_exact = false;
  }
  q.pend = Pending();
  return MM_OK;
}

static int post(mm_engine* e, Queue& q, int64_t cap, const uint64_t* hdr, const int64_t* cookie,
                const int64_t* off, int64_t n) {
  if (!e || n < 0 || (n > 0 && !hdr)) return MM_ERR_ARG;
  if (e->n_ep > 1 && !off) return MM_ERR_ARG;
  const bool off_dev = is_device_ptr(off);
  if (off && !off_dev) {  // host offsets can be validated here
    if (off[0] != 0 || off[e->n_ep] != n) return MM_ERR_ARG;
    for (int i = 0; i < e->n_ep; i++)
      if (off[i + 1] < off[i]) return MM_ERR_ARG;
  }
  int rc = materialize(e, q, cap);
  if (rc != MM_OK) return rc;
  Pending p;
  p.n = n;
  p.seq0 = q.seq;
  p.active = n > 0;
  const int C = pipeline_chunks(e);
  if (n > 0 && C > 1 && off && !off_dev && !is_device_ptr(hdr) && (!cookie || !is_device_ptr(cookie))) {
    // Host input of the MPI level: staged in endpoint ranges on the copy
    // stream, submitted by mm_match_batch (issue_chunks) so that range k of
    // both queues lands first and is matched while k + 1 is in flight.
    CK(ensure(q.st_hdr, (size_t)n * 8));
    if (cookie) CK(ensure(q.st_cookie, (size_t)n * 8));
    CK(ensure(q.st_off, (size_t)(e->n_ep + 1) * 8));
    CK(cudaMemcpyAsync(q.st_off.p, off, (size_t)(e->n_ep + 1) * 8, cudaMemcpyHostToDevice, e->st));
    p.hdr = (const uint64_t*)q.st_hdr.p;
    p.cookie = cookie ? (const int64_t*)q.st_cookie.p : nullptr;
    p.off = (const int64_t*)q.st_off.p;
    p.h_hdr = hdr;
    p.h_cookie = cookie;
    p.h_off = off;
    p.chunks = C;
  } else if (n > 0) {
    if (is_device_ptr(hdr)) {
      p.hdr = hdr;
    } else {
      CK(ensure(q.st_hdr, (size_t)n * 8));
      CK(cudaMemcpyAsync(q.st_hdr.p, hdr, (size_t)n * 8, cudaMemcpyHostToDevice, e->st));
      p.hdr = (const uint64_t*)q.st_hdr.p;
    }
    if (cookie) {
      if (is_device_ptr(cookie)) {
        p.cookie = cookie;
      } else {
        CK(ensure(q.st_cookie, (size_t)n * 8));
        CK(cudaMemcpyAsync(q.st_cookie.p, cookie, (size_t)n * 8, cudaMemcpyHostToDevice, e->st));
        p.cookie = (const int64_t*)q.st_cookie.p;
      }
    }
    if (off) {
      if (off_dev) {
        p.off = off;
      } else {
        CK(ensure(q.st_off, (size_t)(e->n_ep + 1) * 8));
        CK(cudaMemcpyAsync(q.st_off.p, off, (size_t)(e->n_ep + 1) * 8, cudaMemcpyHostToDevice, e->st));
        p.off = (const int64_t*)q.st_off.p;
      }
    }
  }
  if (n > 0 && ((off && !off_dev) || !is_device_ptr(hdr) || (cookie && !is_device_ptr(cookie)))) {
    CK(cudaEventRecord(e->ev_in_st, e->st));
    e->in_st = true;
  }
  q.seq += n;
  q.pend = p;
  return MM_OK;
}

int mm_post_recvs(mm_engine* e, const uint64_t* hdr, const int64_t* cookie, const int64_t* ep_offsets, int64_t n) {
  if (!e) return MM_ERR_ARG;
  LaunchScope ls(e);
  return post(e, e->rq, e->rcap, hdr, cookie, ep_offsets, n);
}

int mm_push_msgs(mm_engine* e, const uint64_t* hdr, const int64_t* cookie, const int64_t* ep_offsets, int64_t n) {
  if (!e) return MM_ERR_ARG;
  LaunchScope ls(e);
  return post(e, e->mq, e->mcap, hdr, cookie, ep_offsets, n);
}

int mm_reset(mm_engine* e) {
  if (!e) return MM_ERR_ARG;
  LaunchScope ls(e);
  // only the current ping-pong buffer (cur = 0) is read before it is written
  CK(launch_reset((int32_t*)e->rq.len[0].p, (int32_t*)e->mq.len[0].p, e->n_ep, (uint32_t*)e->err.p,
                  (unsigned long long*)e->nmatched.p, e->st));
  e->mpi_resid_empty = true;
  e->nm_zero = true;
  e->nm_pending = false;
  Queue* qs[2] = {&e->rq, &e->mq};
  for (Queue* q : qs) {
    q->pend = Pending();
    q->seq = 0;
    q->cur = 0;
    q->resid_host = 0;
    q->resid_exact = true;
  }
  CK(release_host_inputs(e));  // the dropped batch's input copies may still be in flight
  return MM_OK;
}

// Copy device outputs to host outputs / counts when the caller passed host memory.
static int deliver(mm_engine* e, int64_t* out_rc, int64_t* out_mc, bool host_out, int64_t n_copy, int64_t* counts,
                   bool counts_host) {
  if (host_out && n_copy > 0) {
    CK(cudaMemcpyAsync(out_rc, e->out_rc_stage.p, (size_t)n_copy * 8, cudaMemcpyDeviceToHost, e->st));
    CK(cudaMemcpyAsync(out_mc, e->out_mc_stage.p, (size_t)n_copy * 8, cudaMemcpyDeviceToHost, e->st));
  }
  if (counts && counts_host) CK(cudaMemcpyAsync(counts, e->counts_dev.p, 16, cudaMemcpyDeviceToHost, e->st));
  if (host_out || (counts && counts_host)) CK(cudaStreamSynchronize(e->st));
  return MM_OK;
}

static int match_mpi(mm_engine* e, int64_t* out_rc, int64_t* out_mc, int64_t out_cap, int64_t* counts) {
  const bool host_out = !is_device_ptr(out_rc) || !is_device_ptr(out_mc);
  const bool counts_host = counts && !is_device_ptr(counts);
  int64_t* drc = out_rc;
  int64_t* dmc = out_mc;
  // MM_HOST_OUT_MAPPED: page-locked host outputs are written by the kernels
  // directly, through their mapped device addresses (posted PCIe writes
  // while the endpoints are matched: no staging, no D2H copies, no read-back
  // of the output ranges); otherwise host outputs are staged in device
  // memory and copied back.
  int64_t* zrc = host_out && e->host_out == MM_HOST_OUT_MAPPED ? (int64_t*)mapped_host_ptr(out_rc) : nullptr;
  int64_t* zmc = zrc ? (int64_t*)mapped_host_ptr(out_mc) : nullptr;
  const bool zc_out = zrc && zmc;
  if (zc_out) {
    drc = zrc;
    dmc = zmc;
  } else if (host_out) {
    CK(ensure(e->out_rc_stage, (size_t)out_cap * 8));
    CK(ensure(e->out_mc_stage, (size_t)out_cap * 8));
    drc = (int64_t*)e->out_rc_stage.p;
    dmc = (int64_t*)e->out_mc_stage.p;
  }
  const bool staged_out = host_out && !zc_out;
  // Host-buffer pipeline: endpoint range k runs once its H2D chunks landed,
  // and its D2H starts as soon as it finished (H2D, kernels, D2H overlap).
  const int C = pipeline_chunks(e);
  const bool pipe = C > 1 && (staged_out || e->rq.pend.chunks > 0 || e->mq.pend.chunks > 0);
  Queue* qs[2] = {&e->rq, &e->mq};
  if (pipe) {
    Queue* pq[2];
    int np = 0;
    for (Queue* q : qs)
      if (q->pend.chunks == C) pq[np++] = q;
    int ir = issue_chunks(e, pq, np);
    if (ir != MM_OK) return ir;
  }
  for (Queue* q : qs)
    if (!pipe || q->pend.chunks != C) {
      int jr = join_pending(e, *q);
      if (jr != MM_OK) return jr;
    }
  Side R = make_side(e, e->rq, e->rcap), M = make_side(e, e->mq, e->mcap);
  // With no residual receive (after a reset) the snapshot's output offsets
  // are the posted batch's CSR offsets: no scan, and the pair counter was
  // zeroed by mm_reset.  Otherwise one scan, which also zeroes the counter.
  const bool direct = e->mpi_resid_empty && R.p_off && R.p_n <= out_cap;
  const int64_t* out_off = direct ? R.p_off : (const int64_t*)e->out_off.p;
  if (!direct)
    CK(launch_out_offsets(R, e->n_ep, (int64_t*)e->out_off.p, out_cap, (uint32_t*)e->err.p,
                          (unsigned long long*)e->nmatched.p, e->st));
  e->mpi_resid_empty = false;
  // Host outputs: the output ranges are fetched from the device first (staged
  // outputs are copied back by range).  This read-back and wait, before the
  // range kernels are enqueued, also keeps the pipeline overlapped: without
  // it (the caller's host CSR offsets taken instead, or mapped outputs with
  // no read-back) the kernels started only after the whole H2D -- 2.58-2.74
  // vs 1.95-2.0 ms per e2e step on configs[1].
  const int64_t* hoff = e->h_off;
  if (host_out) {
    CK(cudaMemcpyAsync(e->h_off, out_off, (size_t)(e->n_ep + 1) * 8, cudaMemcpyDeviceToHost, e->st));
    CK(cudaStreamSynchronize(e->st));
  }
  MpiArgs a;
  a.R = R;
  a.M = M;
  a.n_ep = e->n_ep;
  a.msg_slots = e->msg_slots;
  a.warp_smem_words = e->warp_words;
  a.out_rc = drc;
  a.out_mc = dmc;
  a.out_cap = out_cap;
  a.out_off = out_off;
  a.q_rh_w = (uint64_t*)e->rq.hdr[0].p;
  a.q_rc_w = (int64_t*)e->rq.cookie[0].p;
  a.rres_w = (int32_t*)e->rq.len[0].p;
  a.q_mh_w = (uint64_t*)e->mq.hdr[0].p;
  a.q_mc_w = (int64_t*)e->mq.cookie[0].p;
  a.mres_w = (int32_t*)e->mq.len[0].p;
  a.n_matched = (unsigned long long*)e->nmatched.p;
  a.err = (uint32_t*)e->err.p;
  const int nchunk = pipe ? C : 1;
  e->timer.begin(e->st);
  for (int k = 0; k < nchunk; k++) {
    a.ep0 = (int)chunk_ep(e, k, nchunk);
    a.n_ep = (int)chunk_ep(e, k + 1, nchunk);
    if (pipe)
      for (Queue* q : qs)
        if (q->pend.active && q->pend.chunks == C) CK(cudaStreamWaitEvent(e->st, q->ev[k], 0));
    if (e->mpi_kernel == MM_MPI_KERNEL_MATRIX)
      CK(launch_mpi_matrix(a, e->st));
    else
      CK(launch_mpi_fifo(a, e->fifo, (uint8_t*)e->fifo_ws.p, e->st));
    if (pipe && staged_out) {
      const int64_t o0 = hoff[a.ep0] < out_cap ? hoff[a.ep0] : out_cap;
      const int64_t o1 = hoff[a.n_ep] < out_cap ? hoff[a.n_ep] : out_cap;
      if (o1 > o0) {
        CK(cudaEventRecord(e->ev_k[k], e->st));
        CK(cudaStreamWaitEvent(e->ds, e->ev_k[k], 0));
        CK(cudaMemcpyAsync(out_rc + o0, drc + o0, (size_t)(o1 - o0) * 8, cudaMemcpyDeviceToHost, e->ds));
        CK(cudaMemcpyAsync(out_mc + o0, dmc + o0, (size_t)(o1 - o0) * 8, cudaMemcpyDeviceToHost, e->ds));
      }
    }
  }
  e->timer.end(e->st);
  CK(launch_finalize(out_off + e->n_ep, 0, (const unsigned long long*)e->nmatched.p, (int64_t*)e->counts_dev.p,
                     counts && !counts_host ? counts : nullptr, e->st));
  e->rq.pend = Pending();
  e->mq.pend = Pending();
  if (pipe) CK(cudaStreamSynchronize(e->cs));  // the caller may reuse its host inputs once we return
  if (pipe && staged_out) {
    CK(cudaStreamSynchronize(e->ds));
    return deliver(e, out_rc, out_mc, false, 0, counts, counts_host);
  }
  if (zc_out) {  // the kernels' writes into the caller's memory are complete once st is
    if (!counts_host) CK(cudaStreamSynchronize(e->st));
    return deliver(e, out_rc, out_mc, false, 0, counts, counts_host);
  }
  const int64_t tot = hoff[e->n_ep];
  return deliver(e, out_rc, out_mc, host_out, host_out ? (tot < out_cap ? tot : out_cap) : 0, counts, counts_host);
}

extern "C++" {
// Capture the launches f(stream) into graph g (appended as root nodes); the
// captured launches are not counted as executed (a conditional body may not
// run).
template <class F>
static cudaError_t capture_into(cudaStream_t gs, cudaGraph_t g, F&& f) {
  cudaError_t err = cudaStreamBeginCaptureToGraph(gs, g, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed);
  if (err != cudaSuccess) return err;
  const long long lc = launch_count();
  const cudaError_t fe = f(gs);
  launch_count() = lc;
  cudaGraph_t out = g;
  err = cudaStreamEndCapture(gs, &out);
  return fe != cudaSuccess ? fe : err;
}

// Append an IF node (after dep) whose body holds the launches of f.
template <class F>
static cudaError_t add_if(cudaStream_t gs, cudaGraph_t g, cudaGraphNode_t dep, cudaGraphConditionalHandle h,
                          cudaGraphNode_t* node, F&& f) {
  cudaGraphNodeParams p = {};
  p.type = cudaGraphNodeTypeConditional;
  p.conditional.handle = h;
  p.conditional.type = cudaGraphCondTypeIf;
  p.conditional.size = 1;
  cudaError_t err = cudaGraphAddNode(node, g, dep ? &dep : nullptr, dep ? 1 : 0, &p);
  if (err != cudaSuccess) return err;
  return capture_into(gs, p.conditional.phGraph_out[0], f);
}

// Append an IF node (after dep) and return its (empty) body graph.
static cudaError_t add_if_body(cudaGraph_t g, cudaGraphNode_t dep, cudaGraphConditionalHandle h, cudaGraphNode_t* node,
                               cudaGraph_t* body) {
  cudaGraphNodeParams p = {};
  p.type = cudaGraphNodeTypeConditional;
  p.conditional.handle = h;
  p.conditional.type = cudaGraphCondTypeIf;
  p.conditional.size = 1;
  cudaError_t err = cudaGraphAddNode(node, g, &dep, 1, &p);
  if (err == cudaSuccess) *body = p.conditional.phGraph_out[0];
  return err;
}

}  // extern "C++"

// The tail of a bucketed no-wildcard batch, decided on the device (one
// graph launch, no host read-back): gate -> IF(overflow) {pair count reset,
// global fallback -- the sort-and-rank over all 64 header bits, or the hash
// table --, both compactions} -> IF(receives partly matched) {slot flags,
// compaction} -> IF(messages partly matched) {slot flags, compaction}; a
// fully matched side's residual queue is emptied by the gate.
static int flat_tail(mm_engine* e, const FlatArgs& a, const BucketScratch& bs, bool ordered, const int64_t res[2],
                     const int64_t ns[2], int64_t* user_counts) {
  Queue* qs[2] = {&e->rq, &e->mq};
  SortScratch ss;
  for (int b = 0; b < 2; b++) {
    ss.key[b] = (uint64_t*)e->skey[b].p;
    ss.val[b] = (uint32_t*)e->sval[b].p;
  }
  ss.rid = (uint32_t*)e->rid.p;
  ss.run_start = (uint32_t*)e->run_start.p;
  ss.run_rc = (uint32_t*)e->run_rc.p;
  ss.part = (uint32_t*)e->part.p;
  ss.scan = (unsigned long long*)e->scan.p;
  HashScratch hs;
  hs.owner = (uint32_t*)e->owner.p;
  hs.rcnt = (uint32_t*)e->rcnt.p;
  hs.mcnt = (uint32_t*)e->mcnt.p;
  hs.tkey = (unsigned long long*)e->tkey.p;
  hs.tval = (uint32_t*)e->tval.p;
  hs.T = next_pow2(2 * a.nr < 1024 ? 1024 : 2 * a.nr);
  mm_engine::TailKey key;
  memset(&key, 0, sizeof(key));
  key.a = a;
  const void* ptrs[] = {bs.bcnt, bs.ix[0], bs.ix[1], bs.sflag[0], bs.sflag[1], bs.overflow,
                        e->rq.hdr[e->rq.cur ^ 1].p, e->rq.cookie[e->rq.cur ^ 1].p, e->rq.len[e->rq.cur ^ 1].p,
                        e->mq.hdr[e->mq.cur ^ 1].p, e->mq.cookie[e->mq.cur ^ 1].p, e->mq.len[e->mq.cur ^ 1].p,
                        e->scan.p, ss.key[0], ss.key[1], ss.val[0], ss.val[1], ss.rid, ss.run_start, ss.run_rc,
                        ss.part, hs.owner, hs.tkey, e->fb_dev.p, e->counts_dev.p, user_counts};
  static_assert(sizeof(ptrs) == sizeof(key.ptr), "TailKey pointers");
  memcpy(key.ptr, ptrs, sizeof(ptrs));
  const int64_t vals[] = {res[0], res[1], ns[0], ns[1], (int64_t)bs.B, ordered ? 1 : 0, hs.T, bs.side_cap};
  memcpy(key.val, vals, sizeof(vals));
  mm_engine::TailGraph* t = nullptr;
  for (auto& c : e->tails)
    if (c.exec && memcmp(&c.key, &key, sizeof(key)) == 0) t = &c;
  if (!t) {  // build: evict the least recently used entry
    t = &e->tails[0];
    for (auto& c : e->tails)
      if (!c.exec || c.stamp < t->stamp) t = &c;
    if (t->exec) cudaGraphExecDestroy(t->exec);
    t->exec = nullptr;
    cudaGraph_t g;
    CK(cudaGraphCreate(&g, 0));
    // h[3]: anything to do at all -- the common all-matched batch evaluates
    // one conditional node (each costs ~9 us of GPU time even when false)
    cudaGraphConditionalHandle h[4];
    cudaError_t err = cudaSuccess;
    for (int i = 0; i < 4 && err == cudaSuccess; i++) err = cudaGraphConditionalHandleCreate(&h[i], g, 0, cudaGraphCondAssignDefault);
    if (err == cudaSuccess)
      err = capture_into(e->gs, g, [&](cudaStream_t st) {
        return launch_flat_gate(bs.overflow, a.n_matched, a.nr, a.nm, h[0], h[1], h[2], h[3],
                                (int32_t*)e->rq.len[e->rq.cur ^ 1].p, (int32_t*)e->mq.len[e->mq.cur ^ 1].p,
                                (unsigned long long*)e->fb_dev.p, (int64_t*)e->counts_dev.p, user_counts, st);
      });
    cudaGraphNode_t prev = nullptr;
    size_t nn = 1;
    if (err == cudaSuccess) err = cudaGraphGetRootNodes(g, &prev, &nn);
    auto compact = [&](int i, const uint8_t* flags, cudaStream_t st) {
      Queue& q = *qs[i];
      const int nb = q.cur ^ 1;
      return run_compact(i ? a.M : a.R, res[i], ns[i], flags, (uint64_t*)q.hdr[nb].p, (int64_t*)q.cookie[nb].p,
                         (int32_t*)q.len[nb].p, (uint32_t*)e->scan.p, st);
    };
    cudaGraphNode_t nany, n0, n1, n2;
    cudaGraph_t body = nullptr;
    if (err == cudaSuccess) err = add_if_body(g, prev, h[3], &nany, &body);
    if (err == cudaSuccess)
      err = add_if(e->gs, body, nullptr, h[0], &n0, [&](cudaStream_t st) {
        cudaError_t r = cudaMemsetAsync(a.n_matched, 0, 8, st);
        if (r == cudaSuccess) r = ordered ? run_sort_rank(a, 0ull, ~0ull, ss, st) : run_hash(a, hs, st);
        if (r == cudaSuccess) r = compact(0, a.rflag, st);
        if (r == cudaSuccess) r = compact(1, a.mflag, st);
        if (r == cudaSuccess)
          r = launch_finalize(nullptr, a.nr, a.n_matched, (int64_t*)e->counts_dev.p, user_counts, st);
        return r;
      });
    for (int i = 0; i < 2 && err == cudaSuccess; i++)
      err = add_if(e->gs, body, i ? n1 : n0, h[1 + i], i ? &n2 : &n1, [&](cudaStream_t st) {
        uint8_t* fl = i ? a.mflag : a.rflag;
        cudaError_t r = run_slot_flags(bs, i, fl, st);
        if (r == cudaSuccess) r = compact(i, fl, st);
        return r;
      });
    if (err == cudaSuccess) err = cudaGraphInstantiate(&t->exec, g, 0);
    cudaGraphDestroy(g);
    if (err != cudaSuccess) {
      t->exec = nullptr;
      cudaGetLastError();
      return MM_ERR_CUDA;
    }
    t->key = key;
  }
  t->stamp = ++e->tail_clock;
  count_launch();  // the gate; the bodies run only when it says so
#if MM_TAIL_SIDE
  // launched on the side stream, ordered by events: a graph launched into the
  // legacy default stream returned only once it had run (a ~27 us gap per
  // step before the next batch's launches)
  CK(cudaEventRecord(e->ev_tail[0], e->st));
  CK(cudaStreamWaitEvent(e->gs, e->ev_tail[0], 0));
  CK(cudaGraphLaunch(t->exec, e->gs));
  CK(cudaEventRecord(e->ev_tail[1], e->gs));
  CK(cudaStreamWaitEvent(e->st, e->ev_tail[1], 0));
#else
  CK(cudaGraphLaunch(t->exec, e->st));
#endif
  return MM_OK;
}

static int match_flat(mm_engine* e, int64_t* out_rc, int64_t* out_mc, int64_t out_cap, int64_t* counts) {
  const bool host_out = !is_device_ptr(out_rc) || !is_device_ptr(out_mc);
  const bool counts_host = counts && !is_device_ptr(counts);
  const bool ordered = e->sem == MM_SEM_NOWILD_ORDERED;
  Side R = make_side(e, e->rq, e->rcap), M = make_side(e, e->mq, e->mcap);
  // the previous device-decided tail has completed (always so when the
  // caller synchronised since, e.g. the sharded path's count exchange): its
  // final pair count is fetched on the side stream -- the engine stream is
  // not waited for -- and the residual sizes are exact again
  if (e->nm_pending && cudaEventQuery(e->ev_nm) == cudaSuccess) {
    e->nm_pending = false;
    CK(cudaMemcpyAsync(&e->h_small->tail_matched, e->nmatched.p, 8, cudaMemcpyDeviceToHost, e->gs));
    CK(cudaStreamSynchronize(e->gs));
    for (Queue* q : {&e->rq, &e->mq}) {
      q->resid_host -= (int64_t)e->h_small->tail_matched;
      q->resid_exact = true;
    }
  }
  cudaGetLastError();  // (a not-yet-complete query is not an error)
  // exact residual sizes (and, for the sort, the varying header bits)
  const int64_t bound = e->rq.resid_host + R.p_n + e->mq.resid_host + M.p_n;
  // the varying header bits (diff) are only needed by the global sort; the
  // residual sizes are read back only when the host does not know them
  bool have_diff = ordered && e->flat_kernel != MM_FLAT_KERNEL_BUCKETED;
  SnapInfo info{};
  if (have_diff || !e->rq.resid_exact || !e->mq.resid_exact) {
    CK(launch_snapshot_info(R, M, bound, (SnapInfo*)e->info.p, have_diff, e->st));
    CK(cudaMemcpyAsync(&e->h_small->info, e->info.p, sizeof(SnapInfo), cudaMemcpyDeviceToHost, e->st));
    CK(cudaStreamSynchronize(e->st));
    info = e->h_small->info;
  } else {
    info.rres = (int32_t)e->rq.resid_host;
    info.mres = (int32_t)e->mq.resid_host;
  }
  const int64_t nr = info.rres + R.p_n, nm = info.mres + M.p_n;
  if (nr > e->rcap || nm > e->mcap) return MM_ERR_CAPACITY;
  if (nr > out_cap) return MM_ERR_CAPACITY;
  int64_t* drc = out_rc;
  int64_t* dmc = out_mc;
  if (host_out) {
    CK(ensure(e->out_rc_stage, (size_t)(nr > 0 ? nr : 1) * 8));
    CK(ensure(e->out_mc_stage, (size_t)(nr > 0 ? nr : 1) * 8));
    drc = (int64_t*)e->out_rc_stage.p;
    dmc = (int64_t*)e->out_mc_stage.p;
  }
  if (!e->nm_zero) CK(cudaMemsetAsync(e->nmatched.p, 0, 8, e->st));
  e->nm_zero = false;
  FlatArgs a;
  a.R = R;
  a.M = M;
  a.nr = nr;
  a.nm = nm;
  a.n_matched = (unsigned long long*)e->nmatched.p;
  a.out_rc = drc;
  a.out_mc = dmc;
  a.rflag = (uint8_t*)e->rflag.p;
  a.mflag = (uint8_t*)e->mflag.p;
  bool done = false;
  unsigned long long matched_host = 0;  // pairs of the bucketed run (valid when done)
  BucketScratch bs;
  if (e->flat_kernel == MM_FLAT_KERNEL_BUCKETED) {
    for (int b = 0; b < 2; b++) {
      bs.h[b] = (uint64_t*)e->bh[b].p;
      bs.ix[b] = (uint32_t*)e->bix[b].p;
      bs.sflag[b] = (uint8_t*)e->bsflag[b].p;
      for (int x = 0; x < 2; x++) {
        bs.xh[x][b] = (uint64_t*)e->bxh[x][b].p;
        bs.xix[x][b] = (uint32_t*)e->bxix[x][b].p;
      }
    }
    bs.cnt = (uint32_t*)e->bcnt.p;
    bs.roff = (uint32_t*)e->broff.p;
    bs.scan = (uint32_t*)e->bscan.p;
    bs.rres = info.rres;
    bs.mres = info.mres;
    e->timer.begin(e->st);
    CK(run_bucketed(a, ordered, bs, e->st));
    e->timer.end(e->st);
    if (e->tail_mode) {
      const int64_t res[2] = {info.rres, info.mres}, ns[2] = {nr, nm};
      const int tr = flat_tail(e, a, bs, ordered, res, ns, counts && !counts_host ? counts : nullptr);
      if (tr != MM_OK) return tr;  // (the tail writes the counts)
      // the residual sizes are known again only if the pair count comes back
      // anyway (host outputs or host counts: the call synchronises)
      // exact residual sizes at once if this call synchronises anyway (host
      // outputs or host counts: the pair count comes back with them), else
      // from the next batch on once this tail has completed (ev_nm)
      const bool back = host_out || counts_host;
      if (back) CK(cudaMemcpyAsync(&e->h_small->tail_matched, e->nmatched.p, 8, cudaMemcpyDeviceToHost, e->st));
      else CK(cudaEventRecord(e->ev_nm, e->st));
      const int dr = deliver(e, out_rc, out_mc, host_out, nr < out_cap ? nr : out_cap, counts, counts_host);
      Queue* qs2[2] = {&e->rq, &e->mq};
      const int64_t ns2[2] = {nr, nm};
      for (int i = 0; i < 2; i++) {
        qs2[i]->cur ^= 1;
        qs2[i]->pend = Pending();
        qs2[i]->resid_host = back ? ns2[i] - (int64_t)e->h_small->tail_matched : ns2[i];
        qs2[i]->resid_exact = back;
      }
      e->nm_pending = !back;
      return dr;
    }
    CK(cudaMemcpyAsync(&e->h_small->over, bs.overflow, 4, cudaMemcpyDeviceToHost, e->st));
    CK(cudaMemcpyAsync(&e->h_small->matched, e->nmatched.p, 8, cudaMemcpyDeviceToHost, e->st));
    CK(cudaStreamSynchronize(e->st));
    matched_host = e->h_small->matched;
    done = e->h_small->over == 0;
    if (!done) {  // a bucket exceeded its region or the on-chip capacity (heavily repeated tuples)
      e->bucket_fallbacks++;
      CK(cudaMemsetAsync(e->nmatched.p, 0, 8, e->st));
    }
  }
  if (!done && ordered && !have_diff) {
    CK(launch_snapshot_info(R, M, bound, (SnapInfo*)e->info.p, true, e->st));
    CK(cudaMemcpyAsync(&e->h_small->info, e->info.p, sizeof(SnapInfo), cudaMemcpyDeviceToHost, e->st));
    CK(cudaStreamSynchronize(e->st));
    info = e->h_small->info;
    have_diff = true;
  }
  if (!done && ordered) {
    SortScratch s;
    for (int b = 0; b < 2; b++) {
      s.key[b] = (uint64_t*)e->skey[b].p;
      s.val[b] = (uint32_t*)e->sval[b].p;
    }
    s.rid = (uint32_t*)e->rid.p;
    s.run_start = (uint32_t*)e->run_start.p;
    s.run_rc = (uint32_t*)e->run_rc.p;
    s.part = (uint32_t*)e->part.p;
    s.scan = (unsigned long long*)e->scan.p;
    e->timer.begin(e->st);
    CK(run_sort_rank(a, info.ref, info.diff, s, e->st));
    e->timer.end(e->st);
  } else if (!done) {
    HashScratch h;
    h.owner = (uint32_t*)e->owner.p;
    h.rcnt = (uint32_t*)e->rcnt.p;
    h.mcnt = (uint32_t*)e->mcnt.p;
    h.tkey = (unsigned long long*)e->tkey.p;
    h.tval = (uint32_t*)e->tval.p;
    h.T = next_pow2(2 * nr < 1024 ? 1024 : 2 * nr);
    e->timer.begin(e->st);
    CK(run_hash(a, h, e->st));
    e->timer.end(e->st);
  }
  // compact both queues into the other ping-pong buffer
  Queue* qs[2] = {&e->rq, &e->mq};
  const Side* ss[2] = {&R, &M};
  const int64_t ns[2] = {nr, nm};
  const int64_t res[2] = {info.rres, info.mres};
  const uint8_t* fl[2] = {a.rflag, a.mflag};
  for (int i = 0; i < 2; i++) {
    Queue& q = *qs[i];
    const int nb = q.cur ^ 1;
    if (done && (int64_t)matched_host == ns[i]) {
      // every element of this side matched (known from the count read back
      // with the overflow flag): the residual queue is empty, no compaction
      CK(cudaMemsetAsync(q.len[nb].p, 0, 4, e->st));
    } else {
      // bucketed: the slots' matched bytes to snapshot order first, so that
      // the residual queue keeps posting / arrival order
      if (done) CK(run_slot_flags(bs, i, (uint8_t*)fl[i], e->st));
      CK(run_compact(*ss[i], res[i], ns[i], fl[i], (uint64_t*)q.hdr[nb].p, (int64_t*)q.cookie[nb].p,
                     (int32_t*)q.len[nb].p, (uint32_t*)e->scan.p, e->st));
    }
    q.cur = nb;
    q.pend = Pending();
    if (done) {  // each pair consumed one element of each side: the residual size is exact
      q.resid_host = ns[i] - (int64_t)matched_host;
      q.resid_exact = true;
    } else {
      q.resid_host = ns[i];  // upper bound until the next exact read
      q.resid_exact = false;
    }
  }
  CK(launch_finalize(nullptr, nr, (const unsigned long long*)e->nmatched.p, (int64_t*)e->counts_dev.p,
                     counts && !counts_host ? counts : nullptr, e->st));
  return deliver(e, out_rc, out_mc, host_out, nr < out_cap ? nr : out_cap, counts, counts_host);
}

int mm_match_batch(mm_engine* e, int64_t* out_recv_cookie, int64_t* out_msg_cookie, int64_t out_capacity,
                   int64_t* counts) {
  if (!e || out_capacity < 0 || (out_capacity > 0 && (!out_recv_cookie || !out_msg_cookie))) return MM_ERR_ARG;
  LaunchScope ls(e);
  const int rc = e->sem == MM_SEM_MPI ? match_mpi(e, out_recv_cookie, out_msg_cookie, out_capacity, counts)
                                      : match_flat(e, out_recv_cookie, out_msg_cookie, out_capacity, counts);
  const cudaError_t wr = release_host_inputs(e);
  return rc != MM_OK ? rc : (wr == cudaSuccess ? MM_OK : MM_ERR_CUDA);
}

int mm_set_option(mm_engine* e, int32_t option, int64_t value) {
  if (!e) return MM_ERR_ARG;
  if (option == MM_OPT_FLAT_KERNEL) {
    if (value != MM_FLAT_KERNEL_BUCKETED && value != MM_FLAT_KERNEL_GLOBAL) return MM_ERR_ARG;
    e->flat_kernel = (int)value;
    return MM_OK;
  }
  if (option == MM_OPT_PIPELINE_CHUNKS) {
    if (value < 0 || value > kMaxChunks) return MM_ERR_ARG;
    e->pipeline = (int)value;
    return MM_OK;
  }
  if (option == MM_OPT_HOST_OUT) {
    if (value != MM_HOST_OUT_STAGED && value != MM_HOST_OUT_MAPPED) return MM_ERR_ARG;
    e->host_out = (int)value;
    return MM_OK;
  }
  if (option == MM_OPT_MPI_KERNEL) {
    if (value == MM_MPI_KERNEL_AUTO) value = MM_MPI_KERNEL_FIFO;
    if (value != MM_MPI_KERNEL_MATRIX && value != MM_MPI_KERNEL_FIFO) return MM_ERR_ARG;
    e->mpi_kernel = (int)value;
    return MM_OK;
  }
  return MM_ERR_ARG;
}

int mm_query(mm_engine* e, int64_t* vals) {
  if (!e || !vals) return MM_ERR_ARG;
  CK(cudaStreamSynchronize(e->st));
  int64_t c[2] = {0, 0};
  CK(cudaMemcpy(c, e->counts_dev.p, 16, cudaMemcpyDeviceToHost));
  uint32_t err = 0;
  CK(cudaMemcpy(&err, e->err.p, 4, cudaMemcpyDeviceToHost));
  int64_t rsum = 0, msum = 0;
  int32_t* tmp = (int32_t*)malloc((size_t)e->n_ep * 4);
  if (!tmp) return MM_ERR_NOMEM;
  CK(cudaMemcpy(tmp, e->rq.len[e->rq.cur].p, (size_t)e->n_ep * 4, cudaMemcpyDeviceToHost));
  for (int i = 0; i < e->n_ep; i++) rsum += tmp[i];
  CK(cudaMemcpy(tmp, e->mq.len[e->mq.cur].p, (size_t)e->n_ep * 4, cudaMemcpyDeviceToHost));
  for (int i = 0; i < e->n_ep; i++) msum += tmp[i];
  free(tmp);
  vals[MM_Q_N_OUT] = c[0];
  vals[MM_Q_N_MATCHED] = c[1];
  vals[MM_Q_RESID_RECV] = rsum;
  vals[MM_Q_RESID_MSG] = msum;
  vals[MM_Q_ERROR] = err;
  e->timer.resolve_all();
  vals[MM_Q_KERNEL_NS] = e->timer.ns;
  vals[MM_Q_KERNEL_RUNS] = e->timer.runs;
  vals[MM_Q_LAUNCHES] = e->launches;
  unsigned long long fbd = 0;
  if (e->fb_dev.p) CK(cudaMemcpy(&fbd, e->fb_dev.p, 8, cudaMemcpyDeviceToHost));
  vals[MM_Q_FALLBACKS] = e->bucket_fallbacks + (int64_t)fbd;
  if (e->sem != MM_SEM_MPI) {
    e->nm_pending = false;
    e->rq.resid_host = rsum;
    e->mq.resid_host = msum;
    e->rq.resid_exact = e->mq.resid_exact = true;
  }
  return err ? MM_ERR_CAPACITY : MM_OK;
}

int mm_route(const uint64_t* a, const int64_t* b, int64_t n, int32_t world, int32_t by, int64_t cookie_base,
             uint64_t* out_a, int64_t* out_b, int64_t* counts, void* stream) {
  if (n < 0 || world < 1 || world > 256 || by < 0 || by > 2 || cookie_base < 0) return MM_ERR_ARG;
  if (by == 2 && (world > 255 || (n > 0 && !b))) return MM_ERR_ARG;
  if (n > 0 && (!a || !out_a || !out_b)) return MM_ERR_ARG;
  const int nc = by == 2 ? 2 * world : world;  // entries of counts
  if (!counts) return MM_ERR_ARG;
  if (n >= ((int64_t)1 << 32)) return MM_ERR_ARG;
  cudaStream_t st = (cudaStream_t)stream;
  if (n > 0 && (!is_device_ptr(a) || !is_device_ptr(out_a) || !is_device_ptr(out_b) || (b && !is_device_ptr(b))))
    return MM_ERR_ARG;
  const bool counts_host = !is_device_ptr(counts);
  void* part = nullptr;
  void* dcounts = nullptr;
  CK(cudaMallocAsync(&part, (size_t)partition_scratch_elems(n > 0 ? n : 1) * 4, st));
  CK(cudaMallocAsync(&dcounts, (size_t)nc * 8, st));
  cudaError_t err = run_route(a, b, n, world, by, cookie_base, out_a, out_b, (int64_t*)dcounts, (uint32_t*)part, st);
  if (err == cudaSuccess)
    err = cudaMemcpyAsync(counts, dcounts, (size_t)nc * 8,
                          counts_host ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice, st);
  cudaFreeAsync(part, st);
  cudaFreeAsync(dcounts, st);
  if (err == cudaSuccess && counts_host) err = cudaStreamSynchronize(st);
  if (err != cudaSuccess) return MM_ERR_CUDA;
  if (counts_host && by != 0) {  // a cookie naming no rank in [0, world) was placed after the groups
    int64_t s = 0;
    for (int w = 0; w < nc; w++) s += counts[w];
    if (s != n) return MM_ERR_ARG;
  }
  return MM_OK;
}

}  // extern "C"
