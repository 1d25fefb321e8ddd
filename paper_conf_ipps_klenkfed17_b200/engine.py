"""Python face of the C-ABI (include/mm.h): the same calls, marshalled.

    eng = Engine(MM_SEM_MPI, n_endpoints=4096, recv_capacity=1024, msg_capacity=1024)
    eng.post_recvs(hdr, cookie=None, ep_offsets=off)     # mm_post_recvs
    eng.push_msgs(hdr, cookie=None, ep_offsets=off)      # mm_push_msgs
    rc, mc = eng.match_batch(out_rc, out_mc)             # mm_match_batch
    eng.reset(); eng.query(); eng.close()                # mm_reset / mm_query / mm_destroy

Arrays may be torch tensors (CUDA or CPU/pinned) or numpy arrays; pointers,
sizes and the current torch CUDA stream are passed through unchanged.  No
matching arithmetic happens in Python.
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import _lib
from ._lib import (MM_NO_MATCH, MM_Q_COUNT, MM_SEM_MPI, MM_SEM_NOWILD_ORDERED,  # noqa: F401
                   MM_SEM_NOWILD_UNORDERED, check)


def _torch():
    import torch
    return torch


def _ptr(x):
    if x is None:
        return None
    if isinstance(x, np.ndarray):
        assert x.flags["C_CONTIGUOUS"]
        return ctypes.c_void_p(x.ctypes.data)
    assert x.is_contiguous(), "tensors must be contiguous"
    return ctypes.c_void_p(x.data_ptr())


def _as_u64(x):
    if isinstance(x, np.ndarray):
        return np.ascontiguousarray(x, dtype=np.uint64)
    torch = _torch()
    if x.dtype == torch.uint64:
        return x.contiguous()
    assert x.dtype == torch.int64, "headers are 64-bit words"
    return x.contiguous()


def _as_i64(x):
    if x is None:
        return None
    if isinstance(x, np.ndarray):
        return np.ascontiguousarray(x, dtype=np.int64)
    torch = _torch()
    assert x.dtype == torch.int64
    return x.contiguous()


def _len(x):
    return int(x.shape[0]) if x is not None else 0


def current_stream_handle(device=None):
    torch = _torch()
    if not torch.cuda.is_available():
        return ctypes.c_void_p(None)  # mm_create then reports MM_ERR_CUDA
    return ctypes.c_void_p(torch.cuda.current_stream(device).cuda_stream)


class Engine:
    """Owns one mm_engine (see include/mm.h for the semantics of each call)."""

    def __init__(self, semantics, n_endpoints=1, recv_capacity=1024, msg_capacity=1024, stream=None,
                 mpi_kernel=None, flat_kernel=None, pipeline_chunks=None, host_out=None):
        L = _lib.load()
        self._L = L
        self.semantics = semantics
        self.n_endpoints = n_endpoints
        self.recv_capacity = recv_capacity
        self.msg_capacity = msg_capacity
        if stream is None:
            stream = current_stream_handle()
        elif not isinstance(stream, ctypes.c_void_p):
            stream = ctypes.c_void_p(stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream))
        self.stream = stream
        self._tstream = None  # torch view of the engine stream (record_stream of device inputs)
        torch = _torch()
        if torch.cuda.is_available():
            self._tstream = (torch.cuda.ExternalStream(stream.value) if stream.value
                             else torch.cuda.default_stream())
        h = ctypes.c_void_p()
        check(L.mm_create(ctypes.byref(h), semantics, n_endpoints, recv_capacity, msg_capacity, stream), "mm_create")
        self._h = h
        self._keep = []  # device buffers referenced by pending batches
        if mpi_kernel is not None:
            self.set_option(_lib.MM_OPT_MPI_KERNEL, mpi_kernel)
        if flat_kernel is not None:
            self.set_option(_lib.MM_OPT_FLAT_KERNEL, flat_kernel)
        if pipeline_chunks is not None:  # MPI level, host buffers: endpoint ranges of the copy pipeline
            self.set_option(_lib.MM_OPT_PIPELINE_CHUNKS, pipeline_chunks)
        if host_out is not None:  # MPI level, host outputs: staged (default) or written in place when page-locked
            self.set_option(_lib.MM_OPT_HOST_OUT, host_out)

    def set_option(self, option, value):
        check(self._L.mm_set_option(self._h, option, value), "mm_set_option")

    def _post(self, fn, name, hdr, cookie, ep_offsets):
        hdr = _as_u64(hdr)
        cookie = _as_i64(cookie)
        ep_offsets = _as_i64(ep_offsets)
        n = _len(hdr)
        check(fn(self._h, _ptr(hdr), _ptr(cookie), _ptr(ep_offsets), n), name)
        # device inputs are read on the engine stream: tell torch's caching
        # allocator, so that a tensor freed after match_batch returns is not
        # reused while the engine stream may still read it
        for t in (hdr, cookie, ep_offsets):
            if self._tstream is not None and t is not None and not isinstance(t, np.ndarray) and t.is_cuda:
                t.record_stream(self._tstream)
        self._keep.append((hdr, cookie, ep_offsets))

    def post_recvs(self, hdr, cookie=None, ep_offsets=None):
        self._post(self._L.mm_post_recvs, "mm_post_recvs", hdr, cookie, ep_offsets)

    def push_msgs(self, hdr, cookie=None, ep_offsets=None):
        self._post(self._L.mm_push_msgs, "mm_push_msgs", hdr, cookie, ep_offsets)

    def match_batch(self, out_rc, out_mc, counts=None):
        """out_rc/out_mc: int64 arrays/tensors of equal length (the capacity).
        counts: optional int64[2] array/tensor receiving {n_out, n_matched}."""
        assert _len(out_rc) == _len(out_mc)
        check(self._L.mm_match_batch(self._h, _ptr(out_rc), _ptr(out_mc), _len(out_rc), _ptr(counts)),
              "mm_match_batch")
        self._keep = []
        return out_rc, out_mc

    def reset(self):
        check(self._L.mm_reset(self._h), "mm_reset")
        self._keep = []

    def query(self, raise_on_error=True):
        vals = np.zeros(MM_Q_COUNT, np.int64)
        rc = self._L.mm_query(self._h, _ptr(vals))
        if raise_on_error:
            check(rc, "mm_query")
        return {"n_out": int(vals[0]), "n_matched": int(vals[1]), "resid_recv": int(vals[2]),
                "resid_msg": int(vals[3]), "error": int(vals[4]), "kernel_ns": int(vals[5]),
                "kernel_runs": int(vals[6]), "launches": int(vals[7]), "fallbacks": int(vals[8]), "rc": rc}

    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            self._L.mm_destroy(self._h)
            self._h = None

    __del__ = close

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()


def route(a, b, world, by, out_a, out_b, counts, stream=None, cookie_base=0):
    """mm_route: stable partition of (a, b) by owner rank (device tensors)."""
    L = _lib.load()
    if stream is None:
        stream = current_stream_handle()
    check(L.mm_route(_ptr(a), _ptr(b), _len(a), world, by, cookie_base, _ptr(out_a), _ptr(out_b), _ptr(counts),
                     stream), "mm_route")
    return out_a, out_b, counts
