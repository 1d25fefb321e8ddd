"""B200-native batched message matching (Klenk et al., IPDPS'17; PAPER.md).

The hot path lives in lib/libmm.so (hand-written sm_100a CUDA behind the
C-ABI of include/mm.h); this package is its Python binding.  See DESIGN.md.
"""
from ._lib import (MM_ANY_SOURCE, MM_ANY_TAG, MM_ERR_ARG, MM_ERR_CAPACITY,  # noqa: F401
                   MM_ERR_CUDA, MM_ERR_NOMEM, MM_ERR_STATE, MM_FLAT_KERNEL_BUCKETED, MM_FLAT_KERNEL_GLOBAL,
                   MM_MPI_KERNEL_FIFO, MM_MPI_KERNEL_MATRIX, MM_MPI_MAX_MSGS, MM_NO_MATCH, MM_OK,
                   MM_HOST_OUT_MAPPED, MM_HOST_OUT_STAGED, MM_OPT_FLAT_KERNEL, MM_OPT_HOST_OUT,
                   MM_OPT_MPI_KERNEL, MM_OPT_PIPELINE_CHUNKS, MM_SEM_MPI,
                   MM_SEM_NOWILD_ORDERED, MM_SEM_NOWILD_UNORDERED, MMError, load, strerror)
from .engine import Engine, route  # noqa: F401

__all__ = ["Engine", "route", "load", "MMError", "MM_SEM_MPI", "MM_SEM_NOWILD_ORDERED",
           "MM_SEM_NOWILD_UNORDERED", "MM_NO_MATCH", "MM_ANY_SOURCE", "MM_ANY_TAG", "MM_OPT_MPI_KERNEL",
           "MM_OPT_FLAT_KERNEL", "MM_OPT_PIPELINE_CHUNKS", "MM_MPI_KERNEL_FIFO", "MM_MPI_KERNEL_MATRIX",
           "MM_FLAT_KERNEL_BUCKETED", "MM_FLAT_KERNEL_GLOBAL", "MM_OPT_HOST_OUT", "MM_HOST_OUT_MAPPED",
           "MM_HOST_OUT_STAGED"]
