"""Seeded synthetic workload generators shared by tests/, bench.py and smoke().

This module holds NO matching arithmetic: it only draws (src, tag, comm)
tuples, places wildcards and lays the queues out in the input format the
C-ABI declares (include/mm.h: one uint64 header word per element, PAPER.md
§IV.A l.115 "the entire header could fit into a single 64-bit word";
per-endpoint CSR offsets).  Both the CPU oracle (oracle/) and the CUDA path
consume what it returns; neither imports the other.

Recipes (stated in DESIGN.md §3 "Input recipe"):

* PAPER.md §IV.A l.113 — most ranks talk to 10–30 peers.
* PAPER.md §IV.A l.115 — tag usage ranges from <4 distinct tags (AMG, LULESH,
  MiniFE) to thousands (MiniDFT, MOCFE, PARTISN); tags fit 16 bits.
* PAPER.md §IV.A l.108 — no application uses ANY_TAG, two use ANY_SOURCE.
* PAPER.md §V.B l.177 — the micro-benchmark queues hold random tuples in
  random order and every message tuple also occurs in the receive queue.
* PAPER.md §VI.C l.221 — the hash-table experiment uses random {src, tag}.
"""
from __future__ import annotations

import numpy as np

ANY_SOURCE = 0xFFFFFFFF
ANY_TAG = 0xFFFF

__all__ = [
    "ANY_SOURCE", "ANY_TAG", "pack", "Queues", "mpi_small", "mpi_endpoints",
    "proxy_endpoints", "nowild_pairs", "worst_chain", "random_case", "widen",
]


def pack(src, tag, comm=0):
    """Header word layout of include/mm.h: src bits 0..31, tag 32..47, comm 48..63."""
    src = np.asarray(src, dtype=np.uint64) & np.uint64(0xFFFFFFFF)
    tag = np.asarray(tag, dtype=np.uint64) & np.uint64(0xFFFF)
    comm = np.asarray(comm, dtype=np.uint64) & np.uint64(0xFFFF)
    return src | (tag << np.uint64(32)) | (comm << np.uint64(48))


class Queues:
    """One batch of input: receive and message headers grouped by endpoint.

    recv_hdr / msg_hdr : uint64 arrays, endpoint-major, each endpoint's
    elements in posting (resp. arrival) order.
    recv_off / msg_off : int64 CSR offsets of length n_endpoints + 1.
    """

    def __init__(self, recv_hdr, recv_off, msg_hdr, msg_off, name=""):
        self.recv_hdr = np.ascontiguousarray(recv_hdr, dtype=np.uint64)
        self.msg_hdr = np.ascontiguousarray(msg_hdr, dtype=np.uint64)
        self.recv_off = np.ascontiguousarray(recv_off, dtype=np.int64)
        self.msg_off = np.ascontiguousarray(msg_off, dtype=np.int64)
        self.name = name
        assert self.recv_off[-1] == len(self.recv_hdr)
        assert self.msg_off[-1] == len(self.msg_hdr)
        assert len(self.recv_off) == len(self.msg_off)

    @property
    def n_endpoints(self):
        return len(self.recv_off) - 1

    def endpoint(self, e):
        return (self.recv_hdr[self.recv_off[e]:self.recv_off[e + 1]],
                self.msg_hdr[self.msg_off[e]:self.msg_off[e + 1]])

    def subset(self, eps):
        """Queues restricted to endpoints `eps` (in the given order)."""
        rs, ms, ro, mo = [], [], [0], [0]
        for e in eps:
            r, m = self.endpoint(int(e))
            rs.append(r), ms.append(m)
            ro.append(ro[-1] + len(r)), mo.append(mo[-1] + len(m))
        cat = lambda xs: np.concatenate(xs) if xs else np.zeros(0, np.uint64)
        return Queues(cat(rs), ro, cat(ms), mo, self.name + "[subset]")


def _wildcard(rng, src, tag, p_any_src, p_any_tag):
    src = src.copy()
    tag = tag.copy()
    src[rng.random(len(src)) < p_any_src] = ANY_SOURCE
    tag[rng.random(len(tag)) < p_any_tag] = ANY_TAG
    return src, tag


def mpi_small(seed=0, n=64, n_src=8, n_tag=16, p_any=0.25):
    """configs[0]: 1 endpoint, 64 posted receives x 64 messages, 8 sources,
    16 tags, 25% ANY_SOURCE and 25% ANY_TAG (drawn independently)."""
    rng = np.random.default_rng(seed)
    msrc = rng.integers(0, n_src, n)
    mtag = rng.integers(0, n_tag, n)
    perm = rng.permutation(n)           # receives: the same tuples, other order
    rsrc, rtag = _wildcard(rng, msrc[perm], mtag[perm], p_any, p_any)
    return Queues(pack(rsrc, rtag), [0, n], pack(msrc, mtag), [0, n], "mpi_small")


def mpi_endpoints(seed, n_ep, depth_r, depth_m=None, n_src=8, n_tag=16,
                  p_any_src=0.25, p_any_tag=0.25, n_comm=1, ragged=False,
                  p_unmatched=0.0):
    """Generic many-endpoint MPI workload used by the parity tests.

    ragged=True draws each endpoint's depths uniformly in [0, depth].
    p_unmatched: fraction of messages whose tuple is redrawn independently of
    the receive queue (so some messages stay unexpected)."""
    rng = np.random.default_rng(seed)
    depth_m = depth_r if depth_m is None else depth_m
    rs, ms, ro, mo = [], [], [0], [0]
    for _ in range(n_ep):
        nr = int(rng.integers(0, depth_r + 1)) if ragged else depth_r
        nm = int(rng.integers(0, depth_m + 1)) if ragged else depth_m
        k = max(nr, nm)
        src = rng.integers(0, n_src, k)
        tag = rng.integers(0, n_tag, k)
        comm = rng.integers(0, n_comm, k)
        mi = rng.permutation(k)[:nm]
        msrc, mtag, mcomm = src[mi], tag[mi], comm[mi]
        redraw = rng.random(nm) < p_unmatched
        msrc[redraw] = rng.integers(0, n_src, int(redraw.sum()))
        mtag[redraw] = rng.integers(0, n_tag, int(redraw.sum()))
        ri = rng.permutation(k)[:nr]
        rsrc, rtag = _wildcard(rng, src[ri], tag[ri], p_any_src, p_any_tag)
        rs.append(pack(rsrc, rtag, comm[ri]))
        ms.append(pack(msrc, mtag, mcomm))
        ro.append(ro[-1] + nr)
        mo.append(mo[-1] + nm)
    return Queues(np.concatenate(rs), ro, np.concatenate(ms), mo, "mpi_endpoints")


def proxy_endpoints(seed=1, n_ep=4096, depth=1024, p_any_src=0.05, p_any_tag=0.0,
                    rank_space=1 << 20):
    """configs[1]: 4096 endpoints x 1024-deep receive and message queues with a
    proxy-app-shaped src/tag mix (§IV.A):

    * each endpoint talks to P ~ U[10, 30] peer ranks drawn from a 2^20 rank
      space (l.113);
    * per endpoint the tag alphabet is drawn from one of three app classes
      (l.115): 'few' (1..4 tags, AMG/LULESH/MiniFE), 'moderate' (16..64),
      'many' (1024..4096 tags, MiniDFT/MOCFE/PARTISN), with weights 1/2, 1/4, 1/4;
    * message tuples are (peer, tag) draws; the receive queue holds the same
      multiset in another random order (every message expected, l.177);
    * ANY_SOURCE on 5% of receives (l.108: only MiniDFT and MiniFE use it),
      no ANY_TAG (l.108: no application uses it); one communicator (l.110).
    """
    rng = np.random.default_rng(seed)
    P = rng.integers(10, 31, n_ep)
    cls = rng.choice(3, n_ep, p=[0.5, 0.25, 0.25])
    ntag = np.where(cls == 0, rng.integers(1, 5, n_ep),
                    np.where(cls == 1, rng.integers(16, 65, n_ep),
                             rng.integers(1024, 4097, n_ep)))
    # vectorised per-endpoint draws
    peer_idx = (rng.random((n_ep, depth)) * P[:, None]).astype(np.int64)
    peers = rng.integers(0, rank_space, (n_ep, 31))
    msrc = np.take_along_axis(peers, peer_idx, axis=1)
    mtag = (rng.random((n_ep, depth)) * ntag[:, None]).astype(np.int64)
    perm = np.argsort(rng.random((n_ep, depth)), axis=1)
    rsrc = np.take_along_axis(msrc, perm, axis=1)
    rtag = np.take_along_axis(mtag, perm, axis=1)
    rsrc = np.where(rng.random((n_ep, depth)) < p_any_src, ANY_SOURCE, rsrc)
    rtag = np.where(rng.random((n_ep, depth)) < p_any_tag, ANY_TAG, rtag)
    off = np.arange(n_ep + 1, dtype=np.int64) * depth
    return Queues(pack(rsrc.ravel(), rtag.ravel()), off,
                  pack(msrc.ravel(), mtag.ravel()), off, "proxy_endpoints")


def nowild_pairs(seed=2, n=1 << 24, n_src=1 << 16, n_tag=64, rank_space=1 << 24,
                 tag_space=1 << 16, n_comm=1, p_unmatched=0.0):
    """configs[2] (n=16M, sort+rank) and configs[3] (hash table) inputs: one
    receive queue and one message queue of n elements each, no wildcards.

    Sources are n_src distinct ranks drawn from rank_space, tags n_tag distinct
    values from tag_space; the message queue is a random permutation of the
    receive tuples (every message expected).  With n_src*n_tag >> n the tuples
    are mostly unique, the regime PAPER.md §VI.C l.217 reports as typical
    (a tuple's share of a destination's messages in the single-digit %).
    p_unmatched redraws that fraction of message tuples independently."""
    rng = np.random.default_rng(seed)
    srcs = rng.choice(rank_space, size=min(n_src, rank_space), replace=False)
    tags = rng.choice(tag_space - 1, size=min(n_tag, tag_space - 1), replace=False)
    src = srcs[rng.integers(0, len(srcs), n)]
    tag = tags[rng.integers(0, len(tags), n)]
    comm = rng.integers(0, n_comm, n)
    rhdr = pack(src, tag, comm)
    mhdr = rhdr[rng.permutation(n)]
    if p_unmatched > 0:
        k = rng.random(n) < p_unmatched
        mhdr[k] = pack(srcs[rng.integers(0, len(srcs), int(k.sum()))],
                       tags[rng.integers(0, len(tags), int(k.sum()))],
                       rng.integers(0, n_comm, int(k.sum())))
    off = np.array([0, n], dtype=np.int64)
    return Queues(rhdr, off, mhdr, off, "nowild_pairs")


def worst_chain(seed=4, depth=16384, n_src=16, n_tag=4, lead_frac=0.25):
    """configs[4]: one endpoint, 16K-deep queues, ANY_SOURCE receives leading.

    The first lead_frac of the receive queue are (ANY_SOURCE, tag) receives;
    the message queue starts with a burst from a single source, so every
    leading wildcard consumes a message some later exact receive of that
    source was also waiting for: each exact receive's earliest admissible
    message sits deep in the queue and the claims form long chains."""
    rng = np.random.default_rng(seed)
    src = rng.integers(0, n_src, depth)
    tag = rng.integers(0, n_tag, depth)
    # message order: sort so that source 0 floods the head of the queue
    order = np.lexsort((rng.random(depth), src != 0))
    msrc, mtag = src[order], tag[order]
    perm = rng.permutation(depth)
    rsrc, rtag = src[perm].copy(), tag[perm].copy()
    lead = int(lead_frac * depth)
    rsrc[:lead] = ANY_SOURCE
    off = np.array([0, depth], dtype=np.int64)
    return Queues(pack(rsrc, rtag), off, pack(msrc, mtag), off, "worst_chain")


def lead_runs(seed, n_ep=1, depth=4096, n_src=12, n_tag=5, lead=1024, kind="src", p_wild_after=0.05,
              msg_frac=1.0, ragged=False):
    """Endpoints whose receive queues START with a run of wildcard receives of
    one type (kind "src": (ANY_SOURCE, tag); "tag": (src, ANY_TAG)) followed
    by exact receives with a p_wild_after share of wildcards of the same type;
    msg_frac < 1 gives fewer messages than receives (some wildcard groups run
    out of messages inside the leading run).  Exercises the global-workspace
    kernel's leading-run path next to the chains."""
    rng = np.random.default_rng(seed)
    rs, ms, ro, mo = [], [], [0], [0]
    for _ in range(n_ep):
        nr = int(rng.integers(depth // 2, depth + 1)) if ragged else depth
        nm = int(msg_frac * nr)
        src = rng.integers(0, n_src, nr)
        tag = rng.integers(0, n_tag, nr)
        mi = rng.permutation(nr)[:nm]
        msrc, mtag = src[mi], tag[mi]
        rsrc, rtag = src.copy(), tag.copy()
        nl = min(lead, nr)
        after = np.zeros(nr, dtype=bool)
        after[nl:] = rng.random(nr - nl) < p_wild_after
        wild = after.copy()
        wild[:nl] = True
        if kind == "src":
            rsrc[wild] = ANY_SOURCE
        else:
            rtag[wild] = ANY_TAG
        rs.append(pack(rsrc, rtag))
        ms.append(pack(msrc, mtag))
        ro.append(ro[-1] + nr)
        mo.append(mo[-1] + nm)
    return Queues(np.concatenate(rs), ro, np.concatenate(ms), mo, "lead_runs")


def random_case(seed, n_ep=3, max_depth=40, wild=True, n_src=4, n_tag=4, n_comm=2):
    """Small irregular case for property tests (ragged depths, empty queues,
    several communicators, optional wildcards, unexpected messages)."""
    rng = np.random.default_rng(seed)
    p = 0.3 if wild else 0.0
    return mpi_endpoints(int(rng.integers(1 << 30)), n_ep, max_depth, n_src=n_src,
                         n_tag=n_tag, p_any_src=p, p_any_tag=p, n_comm=n_comm,
                         ragged=True, p_unmatched=0.2)


def widen(q, seed, p_msg_any_src=0.0, p_msg_any_tag=0.0):
    """The same queues with full-width header fields: every small source id
    is mapped to a distinct random 32-bit value (near-ANY values such as
    0xFFFFFFFE included), every tag to a random 16-bit value (0xFFFE
    included), every communicator to a random 16-bit value; wildcards stay
    wildcards.  p_msg_any_*: fraction of messages that carry the reserved
    wildcard values themselves (matched literally, reading R2).  Only the
    field values change, not which fields are equal."""
    rng = np.random.default_rng(seed)

    def remap(x, width, any_val):
        u = np.unique(x[x != any_val]) if any_val is not None else np.unique(x)
        pool = np.array([(1 << width) - 2, (1 << width) - 3, 0], dtype=np.uint64)
        rand = rng.choice((1 << width) - 1, size=len(u) + 8, replace=False).astype(np.uint64)
        vals = np.unique(np.concatenate([pool, rand]))
        vals = rng.permutation(vals[vals != np.uint64((1 << width) - 1)])[:len(u)]
        out = x.copy()
        if len(u):
            idx = np.searchsorted(u, x)
            keep = (x != any_val) if any_val is not None else np.ones(len(x), bool)
            out[keep] = vals[idx[keep]]
        return out

    def fields(h):
        return h & np.uint64(0xFFFFFFFF), (h >> np.uint64(32)) & np.uint64(0xFFFF), h >> np.uint64(48)

    rs, rt, rc = fields(q.recv_hdr)
    ms, mt, mc = fields(q.msg_hdr)
    nr = len(rs)
    src = remap(np.concatenate([rs, ms]), 32, np.uint64(ANY_SOURCE))
    tag = remap(np.concatenate([rt, mt]), 16, np.uint64(ANY_TAG))
    comm = remap(np.concatenate([rc, mc]), 16, None)
    msrc, mtag = src[nr:], tag[nr:]
    msrc[rng.random(len(msrc)) < p_msg_any_src] = ANY_SOURCE
    mtag[rng.random(len(mtag)) < p_msg_any_tag] = ANY_TAG
    return Queues(pack(src[:nr], tag[:nr], comm[:nr]), q.recv_off, pack(msrc, mtag, comm[nr:]), q.msg_off,
                  q.name + "[wide]")
