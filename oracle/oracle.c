/*
 * oracle/oracle.c -- TEST INFRASTRUCTURE ONLY (not the product path).
 *
 * A plain, slow, obviously-correct CPU oracle for batched message matching
 * as defined in PAPER.md (Klenk, Froening, Eberle, Dennison, "Relaxations for
 * High-Performance Message Passing on Massively Parallel SIMT Processors",
 * IPDPS 2017).  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load it.  It shares no code,
 * header, table or constant generator with the CUDA path under
 * paper_conf_ipps_klenkfed17_b200/ and includes nothing from include/.
 *
 * Functions (each cites the passage it follows):
 *   oracle_mpi_two_list      -- full MPI semantics: the classic posted-receive
 *                               queue / unexpected-message queue traversal
 *                               (§II.B l.65-67).
 *   oracle_nowild_ordered    -- "no source wildcard" relaxation: the rank space
 *                               is partitioned into one queue per source and
 *                               each queue is matched with the same traversal
 *                               (§VI.A l.194-196), wildcard values
 *                               carry no meaning (north_star: "no wildcards
 *                               with per-(src,tag) ordering kept").
 *   oracle_nowild_unordered  -- "no wildcards and ordering": the paper's
 *                               two-level hash table (primary 5x the secondary,
 *                               Jenkins' 32-bit 6-shift hash, colliding
 *                               receives held for the next iteration, unmatched
 *                               messages deferred) (§VI.C l.215-219).
 *   oracle_jenkins32         -- the hash of PAPER.md §VI.C l.219 [17].
 *
 * Header word (the input format, see synth/): src = bits 0..31, tag = bits
 * 32..47, comm = bits 48..63; src 0xFFFFFFFF = MPI_ANY_SOURCE, tag 0xFFFF =
 * MPI_ANY_TAG (only meaningful on receives under full MPI semantics).
 *
 * Pins: tests/test_oracle_pins.py (brute-force enumeration on tiny queues,
 * the paper's own Algorithms 1+2, interleaving invariance, MPI non-overtaking
 * and progress invariants, closed-form rank pairing, per-key match counts).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_ANY_SOURCE 0xFFFFFFFFu
#define ORACLE_ANY_TAG 0xFFFFu

typedef struct {
    uint32_t src, tag, comm;
} tuple_t;

static tuple_t decode(uint64_t h)
{
    tuple_t t;
    t.src = (uint32_t)(h & 0xFFFFFFFFull);
    t.tag = (uint32_t)((h >> 32) & 0xFFFFull);
    t.comm = (uint32_t)((h >> 48) & 0xFFFFull);
    return t;
}

/* PAPER.md §II.B l.65: matching is on (src, tag, comm); the receive may use
 * MPI_ANY_SOURCE for src and MPI_ANY_TAG for tag; comm has no wildcard. */
static int admits_mpi(uint64_t recv, uint64_t msg)
{
    tuple_t r = decode(recv), m = decode(msg);
    if (r.comm != m.comm) return 0;
    if (r.src != ORACLE_ANY_SOURCE && r.src != m.src) return 0;
    if (r.tag != ORACLE_ANY_TAG && r.tag != m.tag) return 0;
    return 1;
}

/* No-wildcard modes: the tuple must be identical (wildcard values literal). */
static int admits_exact(uint64_t recv, uint64_t msg)
{
    tuple_t r = decode(recv), m = decode(msg);
    return r.src == m.src && r.tag == m.tag && r.comm == m.comm;
}

typedef int (*admits_fn)(uint64_t, uint64_t);

/* A doubly linked list over a node pool: the data structure PAPER.md §II.B
 * l.67 names ("Common MPI implementations implement UMQ and PRQ as lists since
 * elements can be easily removed without reordering other elements"). */
typedef struct {
    int64_t *next, *prev;
    int64_t head, tail;
} list_t;

static int list_init(list_t *l, int64_t n)
{
    l->next = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    l->prev = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    l->head = l->tail = -1;
    return (l->next && l->prev) ? 0 : -1;
}

static void list_free(list_t *l)
{
    free(l->next);
    free(l->prev);
}

static void list_append(list_t *l, int64_t x)
{
    l->next[x] = -1;
    l->prev[x] = l->tail;
    if (l->tail >= 0) l->next[l->tail] = x;
    else l->head = x;
    l->tail = x;
}

static void list_unlink(list_t *l, int64_t x)
{
    if (l->prev[x] >= 0) l->next[l->prev[x]] = l->next[x];
    else l->head = l->next[x];
    if (l->next[x] >= 0) l->prev[l->next[x]] = l->prev[x];
    else l->tail = l->prev[x];
}

/*
 * The classic two-list engine on one endpoint (§II.B l.67):
 *  - an incoming receive request looks for a message in the UMQ first; if no
 *    match is found it is appended to the PRQ;
 *  - an incoming message looks for an already posted receive in the PRQ; if
 *    none matches it is kept in the UMQ.
 * Both traversals start at the list head, so the earliest admissible element
 * wins (MPI's in-order guarantee, l.65).
 *
 * recv[0..nr), msg[0..nm): the snapshot of one endpoint in posting / arrival
 * order.  recv[0..nr_resid) and msg[0..nm_resid) are the residual PRQ / UMQ of
 * earlier batches and are in the lists before any event.  `events` orders the
 * new elements: ev >= 0 posts receive ev, ev < 0 delivers message (-ev - 1);
 * events == NULL means "all new messages arrive, then all new receives are
 * posted".  match_r[i] = matched message index or -1, match_m[j] likewise.
 * Returns the number of matched pairs, or -1 on allocation failure or a bad
 * event list.
 */
static int64_t two_list(const uint64_t *recv, int64_t nr, int64_t nr_resid,
                        const uint64_t *msg, int64_t nm, int64_t nm_resid,
                        const int64_t *events, int64_t n_events, admits_fn admits,
                        int64_t *match_r, int64_t *match_m)
{
    list_t prq, umq;
    int64_t matched = 0, i, j, k;
    if (list_init(&prq, nr) || list_init(&umq, nm)) {
        list_free(&prq);
        list_free(&umq);
        return -1;
    }
    for (i = 0; i < nr; i++) match_r[i] = -1;
    for (j = 0; j < nm; j++) match_m[j] = -1;
    for (i = 0; i < nr_resid; i++) list_append(&prq, i);
    for (j = 0; j < nm_resid; j++) list_append(&umq, j);

    int64_t n_ev = events ? n_events : (nm - nm_resid) + (nr - nr_resid);
    for (k = 0; k < n_ev; k++) {
        int64_t ev;
        if (events) ev = events[k];
        else if (k < nm - nm_resid) ev = -(nm_resid + k) - 1;
        else ev = nr_resid + (k - (nm - nm_resid));
        if (ev >= 0) {                       /* a receive is posted */
            i = ev;
            if (i >= nr) { matched = -1; break; }
            for (j = umq.head; j >= 0; j = umq.next[j])
                if (admits(recv[i], msg[j])) break;
            if (j >= 0) {
                list_unlink(&umq, j);
                match_r[i] = j;
                match_m[j] = i;
                matched++;
            } else {
                list_append(&prq, i);
            }
        } else {                             /* a message arrives */
            j = -ev - 1;
            if (j >= nm) { matched = -1; break; }
            for (i = prq.head; i >= 0; i = prq.next[i])
                if (admits(recv[i], msg[j])) break;
            if (i >= 0) {
                list_unlink(&prq, i);
                match_r[i] = j;
                match_m[j] = i;
                matched++;
            } else {
                list_append(&umq, j);
            }
        }
    }
    list_free(&prq);
    list_free(&umq);
    return matched;
}

int64_t oracle_mpi_two_list(const uint64_t *recv, int64_t nr, int64_t nr_resid,
                            const uint64_t *msg, int64_t nm, int64_t nm_resid,
                            const int64_t *events, int64_t n_events,
                            int64_t *match_r, int64_t *match_m)
{
    return two_list(recv, nr, nr_resid, msg, nm, nm_resid, events, n_events,
                    admits_mpi, match_r, match_m);
}

/* Many endpoints at once (CSR offsets), default event order per endpoint,
 * no residuals.  Convenience for large sampled parity checks. */
int64_t oracle_mpi_endpoints(const uint64_t *recv, const int64_t *roff,
                             const uint64_t *msg, const int64_t *moff, int64_t n_ep,
                             int64_t *match_r, int64_t *match_m)
{
    int64_t total = 0, e, i, j;
    for (e = 0; e < n_ep; e++) {
        int64_t r0 = roff[e], nr = roff[e + 1] - roff[e];
        int64_t m0 = moff[e], nm = moff[e + 1] - moff[e];
        int64_t got = two_list(recv + r0, nr, 0, msg + m0, nm, 0, NULL, 0,
                               admits_mpi, match_r + r0, match_m + m0);
        if (got < 0) return -1;
        total += got;
        /* endpoint-local indices -> snapshot-global indices */
        for (i = 0; i < nr; i++)
            if (match_r[r0 + i] >= 0) match_r[r0 + i] += m0;
        for (j = 0; j < nm; j++)
            if (match_m[m0 + j] >= 0) match_m[m0 + j] += r0;
    }
    return total;
}

/* ---------------------------------------------------------------------- */
/* No wildcards, ordering kept: per-source queues (§VI.A l.196,   */
/* "Prohibiting the src wildcard allows the rank space to be statically    */
/* partitioned and arranged into multiple queues").                         */

static const uint64_t *g_sort_keys;
static int cmp_by_src_then_index(const void *a, const void *b)
{
    int64_t x = *(const int64_t *)a, y = *(const int64_t *)b;
    uint32_t sx = (uint32_t)(g_sort_keys[x] & 0xFFFFFFFFull);
    uint32_t sy = (uint32_t)(g_sort_keys[y] & 0xFFFFFFFFull);
    if (sx != sy) return sx < sy ? -1 : 1;
    return x < y ? -1 : (x > y ? 1 : 0);
}

/* Stable grouping of indices by source (a library sort used as one step). */
static int64_t *group_by_src(const uint64_t *h, int64_t n)
{
    int64_t *idx = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    int64_t i;
    if (!idx) return NULL;
    for (i = 0; i < n; i++) idx[i] = i;
    g_sort_keys = h;
    qsort(idx, (size_t)n, sizeof(int64_t), cmp_by_src_then_index);
    return idx;
}

int64_t oracle_nowild_ordered(const uint64_t *recv, int64_t nr, const uint64_t *msg,
                              int64_t nm, int64_t *match_r, int64_t *match_m)
{
    int64_t *ri = group_by_src(recv, nr), *mi = group_by_src(msg, nm);
    int64_t total = 0, a = 0, b = 0, i;
    uint64_t *qr = NULL, *qm = NULL;
    int64_t *lr = NULL, *lm = NULL;
    if (!ri || !mi) goto fail;
    qr = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(nr > 0 ? nr : 1));
    qm = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(nm > 0 ? nm : 1));
    lr = (int64_t *)malloc(sizeof(int64_t) * (size_t)(nr > 0 ? nr : 1));
    lm = (int64_t *)malloc(sizeof(int64_t) * (size_t)(nm > 0 ? nm : 1));
    if (!qr || !qm || !lr || !lm) goto fail;
    for (i = 0; i < nr; i++) match_r[i] = -1;
    for (i = 0; i < nm; i++) match_m[i] = -1;
    /* walk the per-source queues in ascending source order */
    while (a < nr || b < nm) {
        uint32_t s;
        uint32_t sa = a < nr ? (uint32_t)(recv[ri[a]] & 0xFFFFFFFFull) : 0xFFFFFFFFu;
        uint32_t sb = b < nm ? (uint32_t)(msg[mi[b]] & 0xFFFFFFFFull) : 0xFFFFFFFFu;
        int64_t a1 = a, b1 = b, k, n_r, n_m, got;
        if (a >= nr) s = sb;
        else if (b >= nm) s = sa;
        else s = sa < sb ? sa : sb;
        while (a1 < nr && (uint32_t)(recv[ri[a1]] & 0xFFFFFFFFull) == s) a1++;
        while (b1 < nm && (uint32_t)(msg[mi[b1]] & 0xFFFFFFFFull) == s) b1++;
        n_r = a1 - a;
        n_m = b1 - b;
        for (k = 0; k < n_r; k++) qr[k] = recv[ri[a + k]];
        for (k = 0; k < n_m; k++) qm[k] = msg[mi[b + k]];
        got = two_list(qr, n_r, 0, qm, n_m, 0, NULL, 0, admits_exact, lr, lm);
        if (got < 0) goto fail;
        total += got;
        for (k = 0; k < n_r; k++)
            if (lr[k] >= 0) match_r[ri[a + k]] = mi[b + lr[k]];
        for (k = 0; k < n_m; k++)
            if (lm[k] >= 0) match_m[mi[b + k]] = ri[a + lm[k]];
        a = a1;
        b = b1;
        if (n_r == 0 && n_m == 0) break; /* cannot happen; guards the loop */
    }
    free(ri); free(mi); free(qr); free(qm); free(lr); free(lm);
    return total;
fail:
    free(ri); free(mi); free(qr); free(qm); free(lr); free(lm);
    return -1;
}

/* ---------------------------------------------------------------------- */
/* No wildcards, no ordering: two-level hash table (§VI.C l.219). */

/* Robert Jenkins' 32-bit integer hash, the "6-shifts" variant [17]. */
uint32_t oracle_jenkins32(uint32_t a)
{
    a = (a + 0x7ed55d16u) + (a << 12);
    a = (a ^ 0xc761c23cu) ^ (a >> 19);
    a = (a + 0x165667b1u) + (a << 5);
    a = (a + 0xd3a2646cu) ^ (a << 9);
    a = (a + 0xfd7046c5u) + (a << 3);
    a = (a ^ 0xb55a4f09u) ^ (a >> 16);
    return a;
}

/* The paper hashes the {src, tag} tuple with a 32-bit function; the 64-bit
 * word is folded by hashing its high half into its low half (reading R7). */
static uint32_t key_hash(uint64_t h)
{
    return oracle_jenkins32((uint32_t)h ^ oracle_jenkins32((uint32_t)(h >> 32)));
}

static int cmp_u64(const void *a, const void *b)
{
    uint64_t x = *(const uint64_t *)a, y = *(const uint64_t *)b;
    return x < y ? -1 : (x > y ? 1 : 0);
}

static int has_key(const uint64_t *sorted, int64_t n, uint64_t k)
{
    int64_t lo = 0, hi = n;
    while (lo < hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (sorted[mid] < k) lo = mid + 1;
        else hi = mid;
    }
    return lo < n && sorted[lo] == k;
}

/*
 * Iterations of PAPER.md §VI.C l.219:
 *   phase 1: every pending receive is inserted into the primary table; on a
 *            collision into the secondary table; on another collision it is
 *            held for the next iteration;
 *   phase 2: every pending message hashes its key and queries the primary
 *            table, then the secondary; a hit matches (and frees the slot),
 *            otherwise the message is deferred to the next iteration.
 * Sizes: secondary S = max(1, ceil(n_recv / 4)), primary P = 5 S (reading R8).
 * Termination (the paper is silent, reading R9): an iteration that neither
 * inserts nor matches retires the table entries whose key no pending message
 * carries (they can never match in this batch); the loop ends when no pending
 * message is left, or no receive is pending or tabled, or nothing changes.
 */
int64_t oracle_nowild_unordered(const uint64_t *recv, int64_t nr, const uint64_t *msg,
                                int64_t nm, int64_t *match_r, int64_t *match_m,
                                int64_t *n_iterations)
{
    int64_t S = nr > 0 ? (nr + 3) / 4 : 1, P = 5 * S;
    int64_t *prim = (int64_t *)malloc(sizeof(int64_t) * (size_t)P);
    int64_t *sec = (int64_t *)malloc(sizeof(int64_t) * (size_t)S);
    int64_t *pend_r = (int64_t *)malloc(sizeof(int64_t) * (size_t)(nr > 0 ? nr : 1));
    int64_t *pend_m = (int64_t *)malloc(sizeof(int64_t) * (size_t)(nm > 0 ? nm : 1));
    uint64_t *keys = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(nm > 0 ? nm : 1));
    int64_t n_pr = nr, n_pm = nm, total = 0, iters = 0, i, k, tabled = 0;
    if (!prim || !sec || !pend_r || !pend_m || !keys) {
        total = -1;
        goto out;
    }
    for (i = 0; i < P; i++) prim[i] = -1;
    for (i = 0; i < S; i++) sec[i] = -1;
    for (i = 0; i < nr; i++) { pend_r[i] = i; match_r[i] = -1; }
    for (i = 0; i < nm; i++) { pend_m[i] = i; match_m[i] = -1; }

    while (n_pm > 0 && (n_pr > 0 || tabled > 0)) {
        int64_t progress = 0, keep = 0;
        iters++;
        /* phase 1: insert receives */
        for (k = 0; k < n_pr; k++) {
            int64_t r = pend_r[k];
            uint32_t h = key_hash(recv[r]);
            int64_t ps = (int64_t)(h % (uint32_t)P);
            int64_t ss = (int64_t)(oracle_jenkins32(h) % (uint32_t)S);
            if (prim[ps] < 0) { prim[ps] = r; tabled++; progress++; }
            else if (sec[ss] < 0) { sec[ss] = r; tabled++; progress++; }
            else pend_r[keep++] = r;          /* hold for the next iteration */
        }
        n_pr = keep;
        /* phase 2: probe with messages */
        keep = 0;
        for (k = 0; k < n_pm; k++) {
            int64_t m = pend_m[k];
            uint32_t h = key_hash(msg[m]);
            int64_t ps = (int64_t)(h % (uint32_t)P);
            int64_t ss = (int64_t)(oracle_jenkins32(h) % (uint32_t)S);
            int64_t r = -1;
            if (prim[ps] >= 0 && admits_exact(recv[prim[ps]], msg[m])) {
                r = prim[ps];
                prim[ps] = -1;
            } else if (sec[ss] >= 0 && admits_exact(recv[sec[ss]], msg[m])) {
                r = sec[ss];
                sec[ss] = -1;
            }
            if (r >= 0) {
                match_r[r] = m;
                match_m[m] = r;
                total++;
                tabled--;
                progress++;
            } else {
                pend_m[keep++] = m;          /* defer to the next iteration */
            }
        }
        n_pm = keep;
        if (progress == 0 && n_pm > 0) {
            /* retire tabled receives no pending message can ever match */
            int64_t retired = 0;
            for (k = 0; k < n_pm; k++) keys[k] = msg[pend_m[k]];
            qsort(keys, (size_t)n_pm, sizeof(uint64_t), cmp_u64);
            for (i = 0; i < P; i++)
                if (prim[i] >= 0 && !has_key(keys, n_pm, recv[prim[i]])) {
                    prim[i] = -1; tabled--; retired++;
                }
            for (i = 0; i < S; i++)
                if (sec[i] >= 0 && !has_key(keys, n_pm, recv[sec[i]])) {
                    sec[i] = -1; tabled--; retired++;
                }
            if (retired == 0) break;
        }
    }
out:
    if (n_iterations) *n_iterations = iters;
    free(prim); free(sec); free(pend_r); free(pend_m); free(keys);
    return total;
}
