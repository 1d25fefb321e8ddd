"""CPU oracle for batched message matching -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline and
``--impl reference`` legs may import this package.  The product path
(paper_conf_ipps_klenkfed17_b200/) never imports it and shares no code with
it; the only module both sides use is synth/ (seeded inputs, no matching
arithmetic).

The arithmetic lives in oracle.c (plain C, built with gcc by build() or on
first use); this file is ctypes marshalling plus the batch bookkeeping that
the C-ABI defines (residual queues, cookies, endpoint-major output order).

Pins: tests/test_oracle_pins.py.  Parity of every oracle function is pinned
(brute force, the paper's Algorithms 1+2, interleaving invariance, invariants,
closed forms); see DESIGN.md §4.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

SEM_MPI, SEM_NOWILD_ORDERED, SEM_NOWILD_UNORDERED = 0, 1, 2
NO_MATCH = -1


def build(force=False):
    """Compile oracle.c with gcc (plain -O2; never tuned)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-fPIC", "-shared", "-Wall",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        p = ctypes.c_void_p
        i64 = ctypes.c_int64
        L.oracle_mpi_two_list.argtypes = [p, i64, i64, p, i64, i64, p, i64, p, p]
        L.oracle_mpi_two_list.restype = i64
        L.oracle_mpi_endpoints.argtypes = [p, p, p, p, i64, p, p]
        L.oracle_mpi_endpoints.restype = i64
        L.oracle_nowild_ordered.argtypes = [p, i64, p, i64, p, p]
        L.oracle_nowild_ordered.restype = i64
        L.oracle_nowild_unordered.argtypes = [p, i64, p, i64, p, p, p]
        L.oracle_nowild_unordered.restype = i64
        L.oracle_jenkins32.argtypes = [ctypes.c_uint32]
        L.oracle_jenkins32.restype = ctypes.c_uint32
        _lib = L
    return _lib


def _u64(a):
    return np.ascontiguousarray(a, dtype=np.uint64)


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None else None


def mpi_two_list(recv, msg, nr_resid=0, nm_resid=0, events=None):
    """Full MPI semantics on one endpoint (oracle.c: oracle_mpi_two_list).

    events: None (all new messages arrive, then all new receives post) or an
    int64 sequence, ev >= 0 posts receive ev, ev < 0 delivers message -ev-1.
    Returns (match_r, match_m) int64 arrays (-1 = unmatched)."""
    recv, msg = _u64(recv), _u64(msg)
    mr = np.empty(len(recv), np.int64)
    mm = np.empty(len(msg), np.int64)
    ev = None if events is None else np.ascontiguousarray(events, dtype=np.int64)
    n = lib().oracle_mpi_two_list(_ptr(recv), len(recv), nr_resid, _ptr(msg), len(msg),
                                  nm_resid, _ptr(ev), 0 if ev is None else len(ev),
                                  _ptr(mr), _ptr(mm))
    if n < 0:
        raise RuntimeError("oracle_mpi_two_list failed")
    return mr, mm


def mpi_endpoints(q):
    """Full MPI semantics on every endpoint of synth.Queues q (fresh queues).
    Returns snapshot-global (match_r, match_m)."""
    recv, msg = _u64(q.recv_hdr), _u64(q.msg_hdr)
    ro = np.ascontiguousarray(q.recv_off, np.int64)
    mo = np.ascontiguousarray(q.msg_off, np.int64)
    mr = np.empty(len(recv), np.int64)
    mm = np.empty(len(msg), np.int64)
    n = lib().oracle_mpi_endpoints(_ptr(recv), _ptr(ro), _ptr(msg), _ptr(mo),
                                   q.n_endpoints, _ptr(mr), _ptr(mm))
    if n < 0:
        raise RuntimeError("oracle_mpi_endpoints failed")
    return mr, mm


def nowild_ordered(recv, msg):
    """No wildcards, per-(src,tag,comm) ordering (oracle.c: per-source queues)."""
    recv, msg = _u64(recv), _u64(msg)
    mr = np.empty(len(recv), np.int64)
    mm = np.empty(len(msg), np.int64)
    if lib().oracle_nowild_ordered(_ptr(recv), len(recv), _ptr(msg), len(msg),
                                   _ptr(mr), _ptr(mm)) < 0:
        raise RuntimeError("oracle_nowild_ordered failed")
    return mr, mm


def nowild_unordered(recv, msg, return_iterations=False):
    """No wildcards, no ordering (oracle.c: the paper's two-level hash table)."""
    recv, msg = _u64(recv), _u64(msg)
    mr = np.empty(len(recv), np.int64)
    mm = np.empty(len(msg), np.int64)
    it = np.zeros(1, np.int64)
    if lib().oracle_nowild_unordered(_ptr(recv), len(recv), _ptr(msg), len(msg),
                                     _ptr(mr), _ptr(mm), _ptr(it)) < 0:
        raise RuntimeError("oracle_nowild_unordered failed")
    return (mr, mm, int(it[0])) if return_iterations else (mr, mm)


def jenkins32(x):
    return int(lib().oracle_jenkins32(ctypes.c_uint32(x & 0xFFFFFFFF)))


def match(semantics, recv, msg, nr_resid=0, nm_resid=0):
    """Dispatch one endpoint snapshot to the oracle of a semantics level."""
    if semantics == SEM_MPI:
        return mpi_two_list(recv, msg, nr_resid, nm_resid)
    if semantics == SEM_NOWILD_ORDERED:
        return nowild_ordered(recv, msg)
    if semantics == SEM_NOWILD_UNORDERED:
        return nowild_unordered(recv, msg)
    raise ValueError(semantics)


class OracleEngine:
    """The batch API of include/mm.h (mm_post_recvs / mm_push_msgs /
    mm_match_batch / mm_reset), evaluated on the CPU oracle.

    Bookkeeping only: per endpoint the residual posted-receive queue and
    unexpected-message queue (header + cookie) are kept in order; a batch's
    snapshot is residual ++ new (§V l.128: "The UMQ is placed at the
    head of the message queue and the PRQ at the head of the receive request
    queue"); the output lists every snapshot receive endpoint-major in queue
    order with its matched message cookie or -1; matched elements are removed
    and the rest stays in order (the compaction of §V.A l.149)."""

    def __init__(self, semantics, n_endpoints=1):
        self.sem = semantics
        self.n_ep = n_endpoints
        z64 = np.zeros(0, np.uint64)
        zi = np.zeros(0, np.int64)
        self.rq = [(z64, zi) for _ in range(n_endpoints)]
        self.mq = [(z64, zi) for _ in range(n_endpoints)]
        self.pr = [[] for _ in range(n_endpoints)]
        self.pm = [[] for _ in range(n_endpoints)]
        self.rseq = 0
        self.mseq = 0

    def _append(self, pend, hdr, cookie, off, seq):
        hdr = _u64(hdr)
        n = len(hdr)
        if cookie is None:
            cookie = np.arange(seq, seq + n, dtype=np.int64)
        cookie = np.ascontiguousarray(cookie, np.int64)
        off = np.array([0, n], np.int64) if off is None else np.asarray(off, np.int64)
        for e in range(self.n_ep):
            a, b = int(off[e]), int(off[e + 1])
            pend[e].append((hdr[a:b], cookie[a:b]))
        return seq + n

    def post_recvs(self, hdr, cookie=None, ep_offsets=None):
        self.rseq = self._append(self.pr, hdr, cookie, ep_offsets, self.rseq)

    def push_msgs(self, hdr, cookie=None, ep_offsets=None):
        self.mseq = self._append(self.pm, hdr, cookie, ep_offsets, self.mseq)

    def reset(self):
        self.__init__(self.sem, self.n_ep)

    def match_batch(self):
        """Returns (out_recv_cookie, out_msg_cookie) int64 arrays."""
        out_r, out_m = [], []
        for e in range(self.n_ep):
            rh = np.concatenate([self.rq[e][0]] + [p[0] for p in self.pr[e]])
            rc = np.concatenate([self.rq[e][1]] + [p[1] for p in self.pr[e]])
            mh = np.concatenate([self.mq[e][0]] + [p[0] for p in self.pm[e]])
            mc = np.concatenate([self.mq[e][1]] + [p[1] for p in self.pm[e]])
            mr, mm = match(self.sem, rh, mh, len(self.rq[e][0]), len(self.mq[e][0]))
            out_r.append(rc)
            mcook = np.full(len(mr), NO_MATCH, np.int64)
            mcook[mr >= 0] = mc[mr[mr >= 0]]
            out_m.append(mcook)
            self.rq[e] = (rh[mr < 0], rc[mr < 0])
            self.mq[e] = (mh[mm < 0], mc[mm < 0])
            self.pr[e] = []
            self.pm[e] = []
        cat = lambda xs: np.concatenate(xs) if xs else np.zeros(0, np.int64)
        return cat(out_r).astype(np.int64), cat(out_m).astype(np.int64)

    def residual_depths(self):
        return ([len(q[0]) for q in self.rq], [len(q[0]) for q in self.mq])
