"""Multi-GPU sharding of the matching path (DESIGN.md §1 row A6).

* MPI level: endpoints are independent (§VI l.186: "partitions among
  communicators" / endpoints); each rank owns its endpoints and runs its own
  Engine -- no collective on the data path (`split_endpoints`).
* No-wildcard levels: with wildcards prohibited the tuple key space partitions
  (§VI.A l.196).  `ShardedMatcher` hash-partitions receives and
  messages by tuple (mm_route, by=0), moves each to its owner with one NCCL
  all-to-all per side, matches every shard in the owner's Engine, and returns
  each receive's result to its origin rank with a second all-to-all (mm_route,
  by=1 on the origin bits of the cookie).  mm_route is stable and
  all_to_all_single concatenates by source rank, so the owner sees every
  tuple's receives (and messages) in the global order (origin rank, local
  index): the ordered level keeps its per-tuple FIFO across ranks.

The kernels are reached through an `ops` object (CudaOps: the C-ABI); tests
inject a CPU stand-in to exercise this host logic over gloo.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

ORIGIN_SHIFT = 40


def split_endpoints(n_endpoints, world, rank):
    """Contiguous endpoint range [lo, hi) owned by `rank`."""
    per = (n_endpoints + world - 1) // world
    lo = min(n_endpoints, rank * per)
    return lo, min(n_endpoints, lo + per)


class CudaOps:
    """The C-ABI kernels behind the sharded path (device tensors)."""

    def __init__(self):
        from . import engine as _engine
        self._engine = _engine

    def route(self, a, b, world, by, cookie_base):
        n = int(a.shape[0])
        out_a = torch.empty(n, dtype=torch.int64, device=a.device)
        out_b = torch.empty(n, dtype=torch.int64, device=a.device)
        counts = torch.empty(2 * world if by == 2 else world, dtype=torch.int64, device=a.device)
        self._engine.route(a, b, world, by, out_a, out_b, counts, cookie_base=cookie_base)
        return out_a, out_b, counts

    def make_engine(self, semantics, capacity):
        return self._engine.Engine(semantics, 1, capacity, capacity)

    def empty(self, n, like):
        return torch.empty(n, dtype=torch.int64, device=like.device)

    def zeros(self, n, like):
        return torch.zeros(n, dtype=torch.int64, device=like.device)


class ShardedMatcher:
    """One logical no-wildcard matching endpoint spread over the process group.

    Per batch, with NCCL (device tensors end to end), ONE host read-back:

    1. route receives and messages by owner (mm_route by=0, on the device);
    2. all-to-all of a 3-int64 record per rank pair (device): to owner o,
       (#receives for o, #messages for o, #residual receives of o's origin
       held here) -- the last from the previous batch's return route;
    3. one ``.cpu()`` of the sent and received records: every split of the
       forward AND of the return trip is now known on the host;
    4. all-to-all of headers and cookies (receives, messages); the owner
       matches its shard (Engine, device counts);
    5. return route by origin, matched before unmatched (mm_route by=2): its
       counts give each origin's residual receives for the next batch's
       step 2, on the device; all-to-all back to the origins.

    Capacity: the owner's Engine must hold its residual plus the batch.
    """

    def __init__(self, semantics, capacity, group=None, ops=None):
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.ops = ops or CudaOps()
        self.capacity = capacity
        self.engine = self.ops.make_engine(semantics, capacity)
        self._last = None
        self._rseq = 0  # running local indices: cookies stay unique across batches
        self._mseq = 0
        self._ret_counts = None  # by=2 counts of the last return route (device): {matched, residual} per origin
        self.host_syncs = 0      # host read-backs that size the exchanges (1 per batch)
        self._host_coll = dist.get_backend(group) == "gloo"

    def _a2a(self, t, out_splits, in_splits):
        """all_to_all_single of one tensor.  With NCCL the device tensors move
        directly over NVLink; with gloo (CPU tests, or several ranks sharing
        one GPU) they are staged through host memory."""
        n_out = int(sum(out_splits))
        o = self.ops.empty(n_out, t)
        if self._host_coll and t.is_cuda:
            oc = torch.empty(n_out, dtype=t.dtype)
            dist.all_to_all_single(oc, t.cpu(), out_splits, in_splits, group=self.group)
            o.copy_(oc)
        else:
            dist.all_to_all_single(o, t, out_splits, in_splits, group=self.group)
        return o

    def match(self, recv_hdr, msg_hdr):
        """Match one batch.  recv_hdr / msg_hdr: this rank's int64 header words.
        Returns (recv_cookie, msg_cookie) pairs for this rank's receives that
        were in an owner's snapshot (this batch's and earlier unmatched ones):
        cookie = (origin_rank << 40) | running local index (over all batches
        this rank posted); msg_cookie = -1 if unmatched.  Grouped by owner,
        matched before unmatched."""
        W, r = self.world, self.rank
        base = r << ORIGIN_SHIFT
        ra, rb, rcnt = self.ops.route(recv_hdr, None, W, 0, base + self._rseq)
        ma, mb, mcnt = self.ops.route(msg_hdr, None, W, 0, base + self._mseq)
        self._rseq += int(recv_hdr.shape[0])
        self._mseq += int(msg_hdr.shape[0])
        if self._ret_counts is None:
            resid = self.ops.zeros(W, rcnt)
        else:
            resid = self._ret_counts.view(W, 2)[:, 1]
        send = torch.stack([rcnt, mcnt, resid], 1).reshape(-1)
        if self._host_coll and send.is_cuda:
            send = send.cpu()
        recv = torch.empty_like(send)
        dist.all_to_all_single(recv, send, group=self.group)
        rec = torch.cat([send.to(recv.device), recv]).cpu().view(2, W, 3).tolist()  # the host sync
        self.host_syncs += 1
        sent, got = rec
        r_out = [x[0] for x in sent]     # my receives for owner o
        m_out = [x[1] for x in sent]     # my messages for owner o
        resid_here = [x[2] for x in sent]  # residual receives of origin o held here
        r_in = [x[0] for x in got]       # receives origin o sends me
        m_in = [x[1] for x in got]
        resid_there = [x[2] for x in got]  # my residual receives held by owner o
        own_rh = self._a2a(ra, r_in, r_out)
        own_rc = self._a2a(rb, r_in, r_out)
        own_mh = self._a2a(ma, m_in, m_out)
        own_mc = self._a2a(mb, m_in, m_out)
        eng = self.engine
        eng.post_recvs(own_rh, own_rc)
        eng.push_msgs(own_mh, own_mc)
        snap_from = [a + b for a, b in zip(resid_here, r_in)]  # owner snapshot per origin
        n_out = sum(snap_from)
        cap = max(1, n_out)
        out_rc = self.ops.empty(cap, own_rh)
        out_mc = self.ops.empty(cap, own_rh)
        counts = self.ops.empty(2, own_rh)
        eng.match_batch(out_rc, out_mc, counts)
        self._last = counts
        # return trip: every result goes back to the rank that posted the receive
        xa, xb, self._ret_counts = self.ops.route(out_rc[:n_out], out_mc[:n_out], W, 2, 0)
        snap_there = [a + b for a, b in zip(resid_there, r_out)]  # my receives in owner o's snapshot
        back_rc = self._a2a(xa, snap_there, snap_from)
        back_mc = self._a2a(xb, snap_there, snap_from)
        return back_rc, back_mc

    def last_local_matches(self):
        """Pairs matched by this rank's shard in the last batch (reads the
        device counts: synchronises)."""
        return int(self._last[1]) if self._last is not None else None

    def close(self):
        self.engine.close()
