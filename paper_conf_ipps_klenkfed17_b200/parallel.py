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
        counts = torch.empty(world, dtype=torch.int64, device=a.device)
        self._engine.route(a, b, world, by, out_a, out_b, counts, cookie_base=cookie_base)
        return out_a, out_b, counts

    def make_engine(self, semantics, capacity):
        return self._engine.Engine(semantics, 1, capacity, capacity)

    def empty(self, n, like):
        return torch.empty(n, dtype=torch.int64, device=like.device)


class ShardedMatcher:
    """One logical no-wildcard matching endpoint spread over the process group."""

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

    def _exchange(self, tensors, counts):
        """all-to-all of equally split tensors; counts[d] elements go to rank d.
        With NCCL the device tensors are exchanged directly over NVLink; with
        gloo (CPU testing, or several ranks sharing one GPU) they are staged
        through host memory."""
        host = dist.get_backend(self.group) == "gloo"
        send = counts.to(torch.int64)
        if host:
            send = send.cpu()
        recv = torch.empty_like(send)
        dist.all_to_all_single(recv, send, group=self.group)
        splits = torch.stack([send.cpu(), recv.cpu()])  # one host round trip for both
        in_splits = splits[0].tolist()
        out_splits = splits[1].tolist()
        n_out = int(sum(out_splits))
        outs = []
        for t in tensors:
            o = self.ops.empty(n_out, t)
            if host and t.is_cuda:
                oc = torch.empty(n_out, dtype=t.dtype)
                dist.all_to_all_single(oc, t.cpu(), out_splits, in_splits, group=self.group)
                o.copy_(oc)
            else:
                dist.all_to_all_single(o, t, out_splits, in_splits, group=self.group)
            outs.append(o)
        return outs

    def match(self, recv_hdr, msg_hdr):
        """Match one batch.  recv_hdr / msg_hdr: this rank's int64 header words.
        Returns (recv_cookie, msg_cookie) pairs for this rank's receives that
        were in an owner's snapshot: cookie = (origin_rank << 40) | running
        local index (over all batches this rank posted);
        msg_cookie = -1 if unmatched."""
        W, r = self.world, self.rank
        base = r << ORIGIN_SHIFT
        ra, rb, rc = self.ops.route(recv_hdr, None, W, 0, base + self._rseq)
        ma, mb, mc = self.ops.route(msg_hdr, None, W, 0, base + self._mseq)
        self._rseq += int(recv_hdr.shape[0])
        self._mseq += int(msg_hdr.shape[0])
        own_rh, own_rc = self._exchange([ra, rb], rc)
        own_mh, own_mc = self._exchange([ma, mb], mc)
        eng = self.engine
        eng.post_recvs(own_rh, own_rc)
        eng.push_msgs(own_mh, own_mc)
        cap = self.capacity
        out_rc = self.ops.empty(cap, own_rh)
        out_mc = self.ops.empty(cap, own_rh)
        counts = self.ops.empty(2, own_rh)
        eng.match_batch(out_rc, out_mc, counts)
        cnt = counts.cpu()
        n_out, n_matched = int(cnt[0]), int(cnt[1])
        self._last = n_matched
        # return trip: every result goes back to the rank that posted the receive
        xa, xb, xc = self.ops.route(out_rc[:n_out], out_mc[:n_out], W, 1, 0)
        back_rc, back_mc = self._exchange([xa, xb], xc)
        return back_rc, back_mc

    def last_local_matches(self):
        return self._last

    def close(self):
        self.engine.close()
