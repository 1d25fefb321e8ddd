"""Randomised parity sweep of the CUDA path against the CPU oracle.

Each seed draws a whole configuration -- endpoint count, ragged depths,
source/tag/communicator alphabets, wildcard rates of both kinds, unexpected
messages, batch splits with residual queues, host or device buffers, the
host-pipeline range count, the MPI kernel, the no-wildcard kernel family --
so the sweep covers combinations the hand-written cases in
test_parity_gpu.py do not enumerate.  MPI and NOWILD_ORDERED are compared
bit-exactly (per batch); NOWILD_UNORDERED on what is unique (R6).
"""
import numpy as np
import pytest

import oracle
import synth
from _util import check_unordered, check_unordered_per_batch, gpu_batches, oracle_batches, single_batch, split_batches
from test_parity_gpu import assert_exact, assert_same_pairs

pytestmark = pytest.mark.gpu

MPI, ORD, UNO = oracle.SEM_MPI, oracle.SEM_NOWILD_ORDERED, oracle.SEM_NOWILD_UNORDERED


def mpi_config(seed):
    rng = np.random.default_rng(1000 + seed)
    depth = int(rng.choice([1, 7, 32, 33, 100, 257, 700, 1024]))
    cfg = dict(
        n_ep=int(rng.choice([1, 2, 5, 64, 255, 256, 300, 1100])),
        depth_r=depth,
        n_src=int(rng.integers(1, 40)),
        n_tag=int(rng.integers(1, 70)),
        p_any_src=float(rng.choice([0.0, 0.05, 0.3, 0.9])),
        p_any_tag=float(rng.choice([0.0, 0.0, 0.1, 0.5])),
        n_comm=int(rng.integers(1, 4)),
        ragged=bool(rng.random() < 0.7),
        p_unmatched=float(rng.choice([0.0, 0.2, 0.6])),
    )
    if cfg["n_ep"] * depth > 300_000:  # keep the oracle in seconds
        cfg["n_ep"] = max(1, 300_000 // depth)
    run = dict(
        batches=int(rng.integers(1, 4)),
        host=[False, True, "in", "out"][int(rng.integers(0, 4))],
        pipeline=int(rng.choice([0, 1, 2, 5, 32])),
        kern=int(rng.choice([1, 2, 2])),
    )
    return cfg, run


@pytest.mark.parametrize("seed", range(150))
def test_fuzz_mpi(seed):
    cfg, run = mpi_config(seed)
    q = synth.mpi_endpoints(seed, **cfg)
    rng = np.random.default_rng(seed)
    batches = split_batches(q, run["batches"], rng) if run["batches"] > 1 else [
        (q.recv_hdr, np.arange(len(q.recv_hdr), dtype=np.int64), q.recv_off,
         q.msg_hdr, np.arange(len(q.msg_hdr), dtype=np.int64), q.msg_off)]
    cap = cfg["depth_r"] * run["batches"]
    g, qs = gpu_batches(MPI, q.n_endpoints, cap, cap, batches, host=run["host"], mpi_kernel=run["kern"],
                        pipeline=run["pipeline"])
    o, oe = oracle_batches(MPI, q.n_endpoints, batches)
    assert_exact(g, o)
    rr, rm = oe.residual_depths()
    assert qs["error"] == 0 and qs["resid_recv"] == sum(rr) and qs["resid_msg"] == sum(rm), (cfg, run)


def flat_config(seed):
    rng = np.random.default_rng(2000 + seed)
    n = int(rng.choice([0, 1, 2, 31, 1000, 4097, 30000, 120000]))
    kinds = int(rng.integers(0, 3))
    if kinds == 0:  # mostly distinct tuples (§VI.C l.217)
        n_src, n_tag = max(2, n), 64
    elif kinds == 1:  # a few messages per tuple (configs[2] shape)
        n_src, n_tag = max(2, n // 16), 4
    else:  # heavily repeated tuples (long runs, possibly over a bucket's capacity)
        n_src, n_tag = int(rng.integers(1, 6)), int(rng.integers(1, 4))
    return dict(n=n, n_src=n_src, n_tag=n_tag, n_comm=int(rng.integers(1, 3)),
                p_unmatched=float(rng.choice([0.0, 0.1, 0.5]))), int(rng.integers(0, 2)), int(rng.integers(1, 4))


@pytest.mark.parametrize("seed", range(60))
def test_fuzz_ordered(seed):
    cfg, flat, nb = flat_config(seed)
    q = synth.nowild_pairs(seed, **cfg)
    rng = np.random.default_rng(seed)
    batches = split_batches(q, nb, rng) if nb > 1 else single_batch(q)
    n = max(1, cfg["n"])
    host = [False, True, "pinned"][seed % 3]  # device buffers: device-decided tails, deferred residual sizes
    g, qs = gpu_batches(ORD, 1, n, n, batches, flat_kernel=flat, host=host)
    o, _ = oracle_batches(ORD, 1, batches)
    assert_same_pairs(g, o)
    assert qs["error"] == 0


@pytest.mark.parametrize("seed", range(60))
def test_fuzz_unordered(seed):
    cfg, flat, _ = flat_config(seed)
    q = synth.nowild_pairs(seed, **cfg)
    n = max(1, cfg["n"])
    g, qs = gpu_batches(UNO, 1, n, n, single_batch(q), flat_kernel=flat)
    grc, gmc, cnt = g[0]
    assert np.array_equal(np.sort(grc), np.arange(cfg["n"]))
    o, _ = oracle_batches(UNO, 1, single_batch(q))
    orc, omc = o[0]
    om = omc >= 0
    keys, counts = np.unique(q.recv_hdr[orc[om]], return_counts=True)
    check_unordered(q.recv_hdr, q.msg_hdr, grc, gmc, dict(zip(keys.tolist(), counts.tolist())))
    assert int(cnt[1]) == int(om.sum()) and qs["error"] == 0


@pytest.mark.parametrize("seed", range(40))
def test_fuzz_unordered_multibatch(seed):
    """NOWILD_UNORDERED over 2-3 batches with residual queues (the stack
    kernel, the device-decided tail and its deferred residual sizes, the
    fallback for heavily repeated tuples), per batch: valid and maximal."""
    cfg, flat, nb = flat_config(seed + 500)
    q = synth.nowild_pairs(seed + 500, **cfg)
    rng = np.random.default_rng(seed)
    batches = split_batches(q, max(2, nb), rng)
    n = max(1, cfg["n"])
    host = [False, True, "pinned"][seed % 3]
    g, qs = gpu_batches(UNO, 1, n, n, batches, flat_kernel=flat, host=host)
    check_unordered_per_batch(g, batches, q.recv_hdr, q.msg_hdr)
    assert qs["error"] == 0
