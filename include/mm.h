/*
 * mm.h -- C-ABI of the B200-native batched message-matching engine.
 *
 * Implements the matching hot path of Klenk, Froening, Eberle, Dennison,
 * "Relaxations for High-Performance Message Passing on Massively Parallel
 * SIMT Processors" (IPDPS 2017; PAPER.md) at its three semantics levels
 * (Table II):
 *
 *   MM_SEM_MPI               wildcards + ordering (Table II rows 1-2, §V)
 *   MM_SEM_NOWILD_ORDERED    no wildcards, per-tuple ordering (rows 3-4, §VI.A)
 *   MM_SEM_NOWILD_UNORDERED  no wildcards, no ordering (rows 5-6, §VI.C)
 *
 * Plain C types only: pointers may be HOST or DEVICE memory (detected per
 * call with cudaPointerGetAttributes; host buffers are staged through the
 * engine's device buffers inside the call, on the engine's stream).  All
 * calls are asynchronous with respect to the host on the engine's stream
 * unless stated otherwise; device results become valid in stream order.
 *
 * Error behaviour: every call returns MM_OK (0) or an MM_ERR_* code and never
 * aborts.  Argument errors are detected on the host and leave the engine
 * unchanged.  Per-endpoint capacity overflows can only be seen on the device:
 * they set a sticky flag that the next mm_query() reports (MM_ERR_CAPACITY);
 * the affected endpoint's batch is rejected (its receives are reported
 * unmatched, its queues keep their previous contents, the pending elements of
 * that endpoint are dropped).
 */
#ifndef MM_H
#define MM_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ------------------------------------------------------------------ header
 * One 64-bit word per receive request or message (§IV.A l.115:
 * "none of the applications needs tag values longer than 16 bits. Together
 * with the 32-bit value for the source and some bits for the communicator,
 * the entire header could fit into a single 64-bit word"):
 *   bits  0..31  src   (MM_ANY_SOURCE = 0xFFFFFFFF is MPI_ANY_SOURCE)
 *   bits 32..47  tag   (MM_ANY_TAG    = 0xFFFF     is MPI_ANY_TAG)
 *   bits 48..63  comm  (no wildcard, §II.B l.65)
 * Wildcard values only have wildcard meaning on receives under MM_SEM_MPI;
 * everywhere else they are ordinary values compared literally. */
#define MM_ANY_SOURCE 0xFFFFFFFFu
#define MM_ANY_TAG 0xFFFFu

static inline uint64_t mm_header(uint32_t src, uint32_t tag, uint32_t comm)
{
    return (uint64_t)src | ((uint64_t)(tag & 0xFFFFu) << 32) | ((uint64_t)(comm & 0xFFFFu) << 48);
}

/* ------------------------------------------------------------- constants */
enum {
    MM_SEM_MPI = 0,
    MM_SEM_NOWILD_ORDERED = 1,
    MM_SEM_NOWILD_UNORDERED = 2
};

enum {
    MM_OK = 0,
    MM_ERR_ARG = 1,      /* bad argument (null engine, bad sizes, bad semantics) */
    MM_ERR_CUDA = 2,     /* a CUDA runtime call failed */
    MM_ERR_CAPACITY = 3, /* a queue or output buffer was too small (sticky) */
    MM_ERR_NOMEM = 4,    /* device or host allocation failed */
    MM_ERR_STATE = 5     /* call not allowed in the current state */
};

#define MM_NO_MATCH (-1)

/* Query slots of mm_query(). */
enum {
    MM_Q_N_OUT = 0,      /* snapshot receives reported by the last batch */
    MM_Q_N_MATCHED = 1,  /* pairs matched by the last batch */
    MM_Q_RESID_RECV = 2, /* receives left in all posted-receive queues */
    MM_Q_RESID_MSG = 3,  /* messages left in all unexpected-message queues */
    MM_Q_ERROR = 4,      /* sticky device error flags (MM_ERR_CAPACITY if set) */
    MM_Q_KERNEL_NS = 5,  /* cumulative device time (ns, CUDA events) of the dominant
                            kernel region of mm_match_batch since mm_create: the
                            matcher kernel (MPI), the sort-and-rank kernels
                            (NOWILD_ORDERED), the hash kernels (NOWILD_UNORDERED) */
    MM_Q_KERNEL_RUNS = 6,/* number of timed regions behind MM_Q_KERNEL_NS */
    MM_Q_LAUNCHES = 7,   /* cumulative count of this library's kernel launches */
    MM_Q_FALLBACKS = 8,  /* no-wildcard batches that overflowed a bucket and ran the
                            global kernels instead */
    MM_Q_COUNT = 9
};

typedef struct mm_engine mm_engine; /* opaque, owned by the library */

/*
 * mm_create -- allocate an engine on the current CUDA device.
 *   semantics       MM_SEM_*.
 *   n_endpoints     number of independent receiving endpoints (>= 1).  Each
 *                   endpoint has its own posted-receive queue (PRQ) and
 *                   unexpected-message queue (UMQ) (§II.B l.67).
 *                   The no-wildcard levels require n_endpoints == 1 (the
 *                   comm field still separates communicators).
 *   recv_capacity   max receives in one endpoint's batch snapshot (residual
 *                   PRQ + newly posted), > 0; <= MM_MPI_MAX_RECVS under MM_SEM_MPI.
 *   msg_capacity    max messages in one endpoint's snapshot, > 0.  Under
 *                   MM_SEM_MPI one endpoint's messages are staged on chip, so
 *                   msg_capacity <= MM_MPI_MAX_MSGS.
 *   stream          cudaStream_t (as void*) all work is ordered on; NULL =
 *                   the legacy default stream.
 *   out             receives the engine handle (owned; free with mm_destroy).
 */
#define MM_MPI_MAX_MSGS 24576
#define MM_MPI_MAX_RECVS 65534
int mm_create(mm_engine **out, int32_t semantics, int32_t n_endpoints,
              int64_t recv_capacity, int64_t msg_capacity, void *stream);

/*
 * mm_post_recvs / mm_push_msgs -- append a batch of receive requests
 * (posting order) / arrived messages (arrival order) to the endpoints.
 * PAPER.md §II.B l.67: a new receive request looks for a message in the
 * Unexpected Message Queue (UMQ) first, else it is appended to the Posted
 * Receive Queue (PRQ); an arriving message looks in the PRQ, else it joins
 * the UMQ.  Here both are batched: the posted receives and pushed messages
 * wait, in order, behind the residual PRQ / UMQ and are matched together by
 * the next mm_match_batch (§V l.128 treats the UMQ and new arrivals as one
 * queue; by DESIGN.md §2.2 this gives the event-driven result).
 *   hdr         n header words, endpoint-major (all of endpoint 0 first).
 *   cookie      n int64 user handles returned in match results (e.g. request
 *               pointer / payload slot), or NULL: the engine numbers the
 *               elements with a per-engine running sequence (first post = 0).
 *   ep_offsets  n_endpoints + 1 int64 CSR offsets into hdr (ep_offsets[0] =
 *               0, ep_offsets[n_endpoints] = n), or NULL when n_endpoints == 1.
 *   n           number of elements (>= 0).
 * Device buffers are used in place and must stay valid and unchanged until
 * the next mm_match_batch has executed (stream order).  Host buffers are
 * copied by the engine asynchronously (fully so from page-locked memory) and
 * must stay valid and unchanged until the next mm_match_batch (or
 * mm_reset) returns; those calls wait for the copies out of them (not for the
 * matching), so the caller may refill the buffers as soon as they return.  At the MPI level with host hdr AND host ep_offsets the
 * copy is deferred to mm_match_batch and issued in endpoint ranges on an
 * internal copy stream (MM_OPT_PIPELINE_CHUNKS), both queues' range k before
 * range k + 1, so that it overlaps the matching of earlier ranges.  A second
 * post (push) before mm_match_batch moves the pending batch into the queues
 * first.
 */
int mm_post_recvs(mm_engine *e, const uint64_t *hdr, const int64_t *cookie,
                  const int64_t *ep_offsets, int64_t n);
int mm_push_msgs(mm_engine *e, const uint64_t *hdr, const int64_t *cookie,
                 const int64_t *ep_offsets, int64_t n);

/*
 * mm_match_batch -- match every endpoint's snapshot (residual PRQ ++ posted
 * receives, residual UMQ ++ pushed messages; §V l.128), then compact
 * the queues (§V.A l.149).
 *   out_recv_cookie  [out_capacity] receives, for every snapshot receive, its
 *                    cookie.  Order: MPI -- endpoint-major, queue order; the
 *                    no-wildcard levels -- every snapshot receive exactly once
 *                    in an engine-defined order (the hash-bucketed kernels
 *                    report bucket by bucket, grouped by tuple; NOWILD_ORDERED
 *                    keeps receives with equal tuples in posting order);
 *                    residual queues keep posting / arrival order;
 *   out_msg_cookie   [out_capacity] the cookie of the message it matched, or
 *                    MM_NO_MATCH.  Either pointer may be host or device.
 *   out_capacity     length of both arrays; must cover the total snapshot
 *                    receive count (else MM_ERR_CAPACITY is flagged and the
 *                    output is truncated).
 *   counts           NULL or int64[2] (host or device): {n_out, n_matched}.
 * Semantics: MPI -- each receive, in posting order, takes the
 * earliest-arrived unmatched message it admits; NOWILD_ORDERED -- the n-th
 * receive of a tuple takes the n-th message of that tuple; NOWILD_UNORDERED --
 * a maximal pairing of equal tuples.  Results for MPI and NOWILD_ORDERED are
 * deterministic and bit-identical to the CPU oracle.
 * With host output pointers (or host counts) the call synchronises the stream;
 * at the MPI level host outputs are copied back per endpoint range as soon as
 * that range is matched (overlapping the next range's copy-in and matching).
 */
int mm_match_batch(mm_engine *e, int64_t *out_recv_cookie, int64_t *out_msg_cookie,
                   int64_t out_capacity, int64_t *counts);

/* mm_reset -- empty all queues (the PRQ and UMQ of PAPER.md §II.B l.67),
 * drop pending batches, clear error flags and restart cookie sequences.
 * Asynchronous on the engine stream, except that it waits for copies still
 * reading the caller's host input buffers of a dropped batch. */
int mm_reset(mm_engine *e);

/* mm_query -- synchronise the engine's stream and fill host int64
 * vals[MM_Q_COUNT].  Returns MM_ERR_CAPACITY if the sticky flag is set. */
int mm_query(mm_engine *e, int64_t *vals);

/* mm_destroy -- free the engine and its queues (the per-endpoint PRQ / UMQ
 * storage of PAPER.md §II.B l.67; synchronises its stream).  NULL is a no-op. */
int mm_destroy(mm_engine *e);

/*
 * mm_route -- stable partition of n (a, b) pairs by owner rank, used to shard
 * the no-wildcard levels' tuple key space over `world` GPUs (DESIGN.md §1
 * row A6) and to return results to their origin.
 *   by == 0: owner = (hash(a) * world) >> 32, a = header word (key partition;
 *            hash = the Jenkins fold of DESIGN.md reading R7);
 *   by == 1: owner = a >> 40, a = a cookie carrying its origin rank in bits
 *            40..63 (result return trip).  A cookie naming no rank in
 *            [0, world) is placed after every owner's group and is not
 *            counted; with host `counts` the call then returns MM_ERR_ARG
 *            (with device counts, sum(counts) < n tells).
 *   by == 2: as by == 1, each owner's group split in two: first the pairs
 *            whose b != MM_NO_MATCH, then those whose b == MM_NO_MATCH
 *            (a = receive cookie, b = matched message cookie: the return trip
 *            also yields each origin's matched and residual receive counts);
 *            counts then has 2 * world entries {matched, unmatched} per
 *            owner; b must not be NULL; world <= 255.
 *   a           n inputs (device).
 *   b           n inputs (device), or NULL: b[k] = cookie_base + k.  The
 *               sharded path passes cookie_base = (rank << 40) | sequence, so
 *               each cookie names its origin rank and a running local index.
 *   cookie_base see b (>= 0).
 *   out_a/out_b n outputs (device), grouped by owner 0..world-1, each group in
 *               input order.
 *   counts      int64[world] (by == 2: int64[2 world]) (device or host)
 *               elements per owner.
 *   world       1..256.
 *   stream      cudaStream_t as void*.
 * Synchronises the stream only when `counts` is host memory.
 */
int mm_route(const uint64_t *a, const int64_t *b, int64_t n, int32_t world, int32_t by,
             int64_t cookie_base, uint64_t *out_a, int64_t *out_b, int64_t *counts, void *stream);

/*
 * mm_set_option -- engine tuning knobs (host-side, takes effect at the next
 * mm_match_batch).
 *   MM_OPT_MPI_KERNEL: which kernel implements the MPI level --
 *     MM_MPI_KERNEL_FIFO (default, MM_MPI_KERNEL_AUTO): per-tuple FIFO lists,
 *       exact receives resolved by prefix counts, wildcards by a warp search
 *       (DESIGN.md §2.3, §7.2);
 *     MM_MPI_KERNEL_MATRIX: the paper's compatibility-matrix scan/reduce
 *       (§V.A Alg. 1-2) re-designed per warp.
 *   Both produce identical results.  Returns MM_ERR_ARG for unknown options
 *   or values.
 */
enum { MM_OPT_MPI_KERNEL = 1, MM_OPT_FLAT_KERNEL = 2, MM_OPT_PIPELINE_CHUNKS = 3 };
enum { MM_MPI_KERNEL_AUTO = 0, MM_MPI_KERNEL_MATRIX = 1, MM_MPI_KERNEL_FIFO = 2 };
/*   MM_OPT_FLAT_KERNEL: how the no-wildcard levels run --
 *     MM_FLAT_KERNEL_BUCKETED (default): hash-bucketed, one CTA per bucket in
 *       shared memory; a batch with a bucket too large for
 *       the chip (heavily repeated tuples) falls back to the global kernels;
 *     MM_FLAT_KERNEL_GLOBAL: always the global kernels (LSD radix sort-and-rank
 *       for NOWILD_ORDERED, HBM hash table for NOWILD_UNORDERED). */
enum { MM_FLAT_KERNEL_BUCKETED = 0, MM_FLAT_KERNEL_GLOBAL = 1 };
/*   MM_OPT_PIPELINE_CHUNKS: endpoint ranges of the MPI level's host-buffer
 *     pipeline (H2D of range k+1, matching of range k and D2H of range k-1
 *     overlap on three streams): 0 = auto (6 at >= 1024 endpoints, 4 at >= 256, else 1;
 *     ranges grow linearly towards the middle), 1 = off, 2..32 = that many ranges.  Results are identical
 *     for every value; a change applies to the next post. */
/*   MM_OPT_HOST_OUT: how the MPI level delivers results into HOST output
 *     buffers -- MM_HOST_OUT_STAGED (default): written to device staging
 *     buffers and copied back range by range on a copy stream (overlapping
 *     the matching of later ranges); MM_HOST_OUT_MAPPED: page-locked
 *     (pinned / registered) output buffers are written by the matching
 *     kernels directly through their mapped device addresses (PCIe posted
 *     writes; no staging, no D2H copy; pageable buffers stay staged) --
 *     measured no faster on configs[1] (2.0 vs 1.97 ms per e2e step,
 *     DESIGN.md §7.5); it saves the staging buffers.  Results are identical; mm_match_batch returns once they
 *     are in host memory either way. */
enum { MM_OPT_HOST_OUT = 4 };
enum { MM_HOST_OUT_STAGED = 0, MM_HOST_OUT_MAPPED = 1 };
int mm_set_option(mm_engine *e, int32_t option, int64_t value);

/* mm_strerror -- static description of an MM_* code. */
const char *mm_strerror(int code);

/* mm_version -- "mm <semver> sm_100a". */
const char *mm_version(void);

#ifdef __cplusplus
}
#endif

#endif /* MM_H */
