"""Parity of the CUDA path (through the C-ABI) with the CPU oracle.

MPI and NOWILD_ORDERED: bit-exact, element by element (receive cookie and
matched message cookie for every snapshot receive, per batch).
NOWILD_UNORDERED: what is unique (reading R6) -- equal tuples per
pair, every message used once, per-tuple counts equal to the oracle's.
"""
import numpy as np
import pytest

import oracle
import synth
from _util import (check_unordered, check_unordered_per_batch, gpu_batches, oracle_batches, per_key_min, per_key_min_np,
                   single_batch,
                   split_batches)

pytestmark = pytest.mark.gpu

MPI, ORD, UNO = oracle.SEM_MPI, oracle.SEM_NOWILD_ORDERED, oracle.SEM_NOWILD_UNORDERED
KERNELS = pytest.mark.parametrize("kern", [1, 2], ids=["matrix", "fifo"])  # MM_MPI_KERNEL_*
FLAT = pytest.mark.parametrize("flat", [0, 1], ids=["bucketed", "global"])  # MM_FLAT_KERNEL_*


def assert_exact(g, o):
    assert len(g) == len(o)
    for b, ((grc, gmc, cnt), (orc, omc)) in enumerate(zip(g, o)):
        assert len(grc) == len(orc), "batch %d: snapshot sizes differ" % b
        assert np.array_equal(grc, orc), "batch %d: receive order differs" % b
        bad = np.nonzero(gmc != omc)[0]
        assert len(bad) == 0, "batch %d: %d mismatches, first at %s: gpu %s oracle %s" % (
            b, len(bad), bad[:5], gmc[bad[:5]], omc[bad[:5]])
        assert int(cnt[1]) == int((omc >= 0).sum())


def assert_same_pairs(g, o):
    """No-wildcard levels report receives in an engine-defined order: compare
    the receive->message map per batch (bit-exact as a map)."""
    assert len(g) == len(o)
    for b, ((grc, gmc, cnt), (orc, omc)) in enumerate(zip(g, o)):
        assert len(grc) == len(orc), "batch %d: snapshot sizes differ" % b
        assert len(np.unique(grc)) == len(grc), "batch %d: a receive reported twice" % b
        gm = dict(zip(grc.tolist(), gmc.tolist()))
        om = dict(zip(orc.tolist(), omc.tolist()))
        assert set(gm) == set(om), "batch %d: different receives" % b
        bad = [k for k in om if gm[k] != om[k]]
        assert not bad, "batch %d: %d mismatches, e.g. recv %s: gpu %s oracle %s" % (
            b, len(bad), bad[0], gm[bad[0]], om[bad[0]])
        assert int(cnt[1]) == int((omc >= 0).sum())


@KERNELS
def test_mpi_config0(kern):
    q = synth.mpi_small(0)
    g, _ = gpu_batches(MPI, 1, 64, 64, single_batch(q), mpi_kernel=kern)
    o, _ = oracle_batches(MPI, 1, single_batch(q))
    assert_exact(g, o)


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("depth", [1, 31, 33, 200, 1024])
@KERNELS
def test_mpi_ragged_endpoints(seed, depth, kern):
    q = synth.mpi_endpoints(seed, n_ep=37, depth_r=depth, n_src=5, n_tag=4, p_any_src=0.3, p_any_tag=0.3,
                            n_comm=2, ragged=True, p_unmatched=0.2)
    g, qs = gpu_batches(MPI, q.n_endpoints, depth, depth, single_batch(q), mpi_kernel=kern)
    o, _ = oracle_batches(MPI, q.n_endpoints, single_batch(q))
    assert_exact(g, o)
    assert qs["error"] == 0


@pytest.mark.parametrize("seed", range(4))
@KERNELS
def test_mpi_multibatch_residuals(seed, kern):
    rng = np.random.default_rng(seed)
    q = synth.mpi_endpoints(seed + 10, n_ep=50, depth_r=150, n_src=4, n_tag=3, p_any_src=0.25, p_any_tag=0.25,
                            ragged=True, p_unmatched=0.3)
    batches = split_batches(q, 4, rng)
    g, qs = gpu_batches(MPI, q.n_endpoints, 600, 600, batches, mpi_kernel=kern)
    o, oe = oracle_batches(MPI, q.n_endpoints, batches)
    assert_exact(g, o)
    rr, rm = oe.residual_depths()
    assert qs["resid_recv"] == sum(rr) and qs["resid_msg"] == sum(rm)


@KERNELS
def test_mpi_host_buffers_equal_device(kern):
    q = synth.mpi_endpoints(5, n_ep=64, depth_r=128, ragged=True, p_unmatched=0.1)
    gd, _ = gpu_batches(MPI, q.n_endpoints, 128, 128, single_batch(q), mpi_kernel=kern)
    gh, _ = gpu_batches(MPI, q.n_endpoints, 128, 128, single_batch(q), host=True, mpi_kernel=kern)
    o, _ = oracle_batches(MPI, q.n_endpoints, single_batch(q))
    assert_exact(gd, o)
    assert_exact(gh, o)


@pytest.mark.parametrize("chunks", [0, 1, 2, 3, 7, 32])
@pytest.mark.parametrize("host", [True, "in", "out", "pinned", "pinned-mapped"],
                         ids=["host-io", "host-in", "host-out", "pinned", "pinned-mapped"])
@KERNELS
def test_mpi_host_pipeline(chunks, host, kern):
    """Host-buffer pipeline (MM_OPT_PIPELINE_CHUNKS): endpoint ranges copied in,
    matched and copied out on three streams; 3 batches with residuals, user
    cookies, ragged and empty endpoints -- identical to the oracle for every
    range count."""
    rng = np.random.default_rng(chunks)
    q = synth.mpi_endpoints(40 + chunks, n_ep=301, depth_r=96, n_src=6, n_tag=4, p_any_src=0.2, p_any_tag=0.1,
                            ragged=True, p_unmatched=0.25)
    batches = split_batches(q, 3, rng)  # carries user cookies (global element ids)
    g, qs = gpu_batches(MPI, q.n_endpoints, 300, 300, batches, host=host, mpi_kernel=kern, pipeline=chunks)
    o, oe = oracle_batches(MPI, q.n_endpoints, batches)
    assert_exact(g, o)
    rr, rm = oe.residual_depths()
    assert qs["error"] == 0 and qs["resid_recv"] == sum(rr) and qs["resid_msg"] == sum(rm)


@pytest.mark.parametrize("host", [True, "pinned", "pinned-mapped"], ids=["pageable", "pinned", "pinned-mapped"])
def test_mpi_host_pipeline_truncated_output(host):
    """A host output too small for the snapshot: the capacity flag is raised
    and the delivered prefix is still the oracle's (page-locked outputs are
    written in place: nothing beyond the capacity is touched)."""
    q = synth.mpi_endpoints(77, n_ep=260, depth_r=64, ragged=True, p_unmatched=0.1)
    o, _ = oracle_batches(MPI, q.n_endpoints, single_batch(q))
    cap = len(o[0][0]) // 2
    g, qs = gpu_batches(MPI, q.n_endpoints, 64, 64, single_batch(q), host=host, out_cap=cap, pipeline=4)
    assert qs["error"] != 0
    # endpoints whose output range fits are reported exactly; the rest is
    # flagged and its output positions are unspecified
    fit = int(q.recv_off[np.searchsorted(q.recv_off, cap, side="right") - 1])
    assert fit > 0
    assert np.array_equal(g[0][0][:fit], o[0][0][:fit]) and np.array_equal(g[0][1][:fit], o[0][1][:fit])


@pytest.mark.parametrize("chunks", [3, 6])
def test_mpi_host_pipeline_two_posts_and_reset(chunks):
    """Deferred host inputs: a second post before the match moves the first
    (its chunk copies are issued and joined first); a reset drops a deferred
    post without copying it; host outputs come back per range."""
    rng = np.random.default_rng(5)
    q = synth.mpi_endpoints(15, n_ep=300, depth_r=40, n_src=5, n_tag=3, p_any_src=0.3, p_any_tag=0.2,
                            ragged=True, p_unmatched=0.2)
    b1, b2 = split_batches(q, 2, rng)
    from paper_conf_ipps_klenkfed17_b200 import Engine
    from paper_conf_ipps_klenkfed17_b200._lib import MM_OPT_PIPELINE_CHUNKS
    eng = Engine(MPI, q.n_endpoints, 80, 80)
    eng.set_option(MM_OPT_PIPELINE_CHUNKS, chunks)
    junk = synth.mpi_endpoints(99, n_ep=300, depth_r=40, ragged=True)
    eng.post_recvs(junk.recv_hdr.astype(np.uint64), None, junk.recv_off)  # dropped by the reset
    eng.reset()
    for (rh, rc, ro, mh, mc, mo) in (b1, b2):  # both halves posted before one match
        eng.post_recvs(np.ascontiguousarray(rh, np.uint64), rc, ro)
        eng.push_msgs(np.ascontiguousarray(mh, np.uint64), mc, mo)
    cap = q.n_endpoints * 80
    orc = np.full(cap, -7, np.int64)
    omc = np.full(cap, -7, np.int64)
    cnt = np.zeros(2, np.int64)
    eng.match_batch(orc, omc, cnt)
    qs = eng.query()
    eng.close()
    oe = oracle.OracleEngine(MPI, q.n_endpoints)
    for (rh, rc, ro, mh, mc, mo) in (b1, b2):
        oe.post_recvs(rh, rc, ro)
        oe.push_msgs(mh, mc, mo)
    o_rc, o_mc = oe.match_batch()
    n = int(cnt[0])
    assert n == len(o_rc) and qs["error"] == 0
    assert np.array_equal(orc[:n], o_rc) and np.array_equal(omc[:n], o_mc)


@KERNELS
def test_mpi_user_cookies_and_two_posts(kern):
    """Cookies are carried through; a second post before a match is queued."""
    q = synth.mpi_endpoints(6, n_ep=8, depth_r=64, p_unmatched=0.1)
    rng = np.random.default_rng(0)
    rc = rng.integers(0, 1 << 50, len(q.recv_hdr))
    mc = rng.integers(0, 1 << 50, len(q.msg_hdr))
    half_r = q.recv_off // 2
    # post each endpoint's first half, then the second half, then match once
    def halves(off, hdr, ck):
        a_idx = np.concatenate([np.arange(off[e], off[e] + (off[e + 1] - off[e]) // 2) for e in range(8)])
        b_idx = np.concatenate([np.arange(off[e] + (off[e + 1] - off[e]) // 2, off[e + 1]) for e in range(8)])
        ao = np.r_[0, np.cumsum([(off[e + 1] - off[e]) // 2 for e in range(8)])]
        bo = np.r_[0, np.cumsum([(off[e + 1] - off[e]) - (off[e + 1] - off[e]) // 2 for e in range(8)])]
        return (hdr[a_idx], ck[a_idx], ao), (hdr[b_idx], ck[b_idx], bo)
    (ra, rb) = halves(q.recv_off, q.recv_hdr, rc)
    (ma, mb) = halves(q.msg_off, q.msg_hdr, mc)
    del half_r
    import torch
    from _util import to_dev
    from paper_conf_ipps_klenkfed17_b200 import Engine
    eng = Engine(MPI, 8, 64, 64, mpi_kernel=kern)
    eng.post_recvs(to_dev(ra[0]), to_dev(ra[1]), to_dev(ra[2]))
    eng.push_msgs(to_dev(ma[0]), to_dev(ma[1]), to_dev(ma[2]))
    eng.post_recvs(to_dev(rb[0]), to_dev(rb[1]), to_dev(rb[2]))
    eng.push_msgs(to_dev(mb[0]), to_dev(mb[1]), to_dev(mb[2]))
    orc = torch.empty(8 * 64, dtype=torch.int64, device="cuda")
    omc = torch.empty_like(orc)
    cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
    eng.match_batch(orc, omc, cnt)
    n = int(cnt[0])
    oe = oracle.OracleEngine(MPI, 8)
    oe.post_recvs(*ra)
    oe.push_msgs(*ma)
    oe.post_recvs(*rb)
    oe.push_msgs(*mb)
    o_rc, o_mc = oe.match_batch()
    assert np.array_equal(orc[:n].cpu().numpy(), o_rc)
    assert np.array_equal(omc[:n].cpu().numpy(), o_mc)
    eng.close()


@KERNELS
def test_mpi_empty_and_degenerate(kern):
    # no receives at all, no messages at all, both empty
    for nr, nm in [(0, 10), (10, 0), (0, 0)]:
        rh = synth.pack(np.arange(nr) % 3, np.zeros(nr, int))
        mh = synth.pack(np.arange(nm) % 3, np.zeros(nm, int))
        b = [(rh, None, np.array([0, nr]), mh, None, np.array([0, nm]))]
        g, _ = gpu_batches(MPI, 1, 16, 16, b, mpi_kernel=kern)
        o, _ = oracle_batches(MPI, 1, b)
        assert_exact(g, o)
    # all (ANY, ANY) receives against many senders
    rh = synth.pack(np.full(100, synth.ANY_SOURCE), np.full(100, synth.ANY_TAG))
    mh = synth.pack(np.arange(90) % 7, np.arange(90) % 5)
    b = [(rh, None, np.array([0, 100]), mh, None, np.array([0, 90]))]
    g, _ = gpu_batches(MPI, 1, 128, 128, b, mpi_kernel=kern)
    o, _ = oracle_batches(MPI, 1, b)
    assert_exact(g, o)


@KERNELS
def test_mpi_capacity_overflow_is_flagged(kern):
    q = synth.mpi_endpoints(3, n_ep=4, depth_r=40)
    g, qs = gpu_batches(MPI, 4, 32, 32, single_batch(q), out_cap=4 * 40, mpi_kernel=kern)
    assert qs["error"] != 0 and qs["rc"] == 3


@KERNELS
def test_mpi_config4_worst_chain(kern):
    q = synth.worst_chain()
    g, _ = gpu_batches(MPI, 1, 16384, 16384, single_batch(q), mpi_kernel=kern)
    o, _ = oracle_batches(MPI, 1, single_batch(q))
    assert_exact(g, o)


@KERNELS
@pytest.mark.parametrize("seed,p_any", [(1, 0.0), (2, 0.1), (3, 0.3)])
def test_mpi_wide_headers_and_literal_any(kern, seed, p_any):
    """Full-width header fields (32-bit src, 16-bit tag and comm, values next
    to the wildcard ones) and messages carrying the reserved ANY values
    (reading R2), ragged endpoints, both wildcard kinds, two communicators,
    unexpected messages, 3 batches with residual queues -- bit-exact."""
    rng = np.random.default_rng(seed)
    q = synth.widen(synth.mpi_endpoints(seed, n_ep=40, depth_r=300, n_src=12, n_tag=6, n_comm=2, ragged=True,
                                        p_unmatched=0.2, p_any_src=0.2, p_any_tag=0.15),
                    seed, p_msg_any_src=p_any, p_msg_any_tag=p_any)
    batches = split_batches(q, 3, rng)
    g, st = gpu_batches(MPI, 40, 300, 300, batches, mpi_kernel=kern)
    o, _ = oracle_batches(MPI, 40, batches)
    assert_exact(g, o)
    assert st["error"] == 0


@pytest.mark.parametrize("kind", ["src", "tag"])
def test_mpi_wide_headers_deep_endpoint(kind):
    """The deep-endpoint (global workspace, 1024-thread) variant on wide
    headers with a leading wildcard run and literal-ANY messages."""
    q = synth.widen(synth.lead_runs(5, n_ep=1, depth=6000, lead=1500, kind=kind, n_src=20, n_tag=6),
                    5, p_msg_any_src=0.05, p_msg_any_tag=0.05)
    g, st = gpu_batches(MPI, 1, 6000, 6000, single_batch(q))
    o, _ = oracle_batches(MPI, 1, single_batch(q))
    assert_exact(g, o)


@pytest.mark.parametrize("host,pipeline", [(False, None), (True, 2), ("in", 3)])
@pytest.mark.parametrize("seed", [1, 2])
def test_mpi_cluster_endpoints_multibatch(seed, host, pipeline):
    """Deep endpoints on the thread-block-cluster variant (few endpoints,
    queues too deep for one CTA's shared memory): ragged depths up to 3000,
    both wildcard kinds, two communicators, unexpected messages, 3 batches
    with residual queues; device buffers and the host-buffer pipeline (the
    cluster kernel launched per endpoint range).  Bit-exact."""
    rng = np.random.default_rng(seed)
    q = synth.mpi_endpoints(seed + 40, n_ep=7, depth_r=3000, n_src=30, n_tag=9, p_any_src=0.08, p_any_tag=0.05,
                            n_comm=2, ragged=True, p_unmatched=0.2)
    batches = split_batches(q, 3, rng)
    g, st = gpu_batches(MPI, 7, 3000, 3000, batches, host=host, pipeline=pipeline)
    o, _ = oracle_batches(MPI, 7, batches)
    assert_exact(g, o)
    assert st["error"] == 0


def test_mpi_cluster_capacity_overflow():
    """Capacity overflow on the cluster variant: an endpoint over capacity is
    flagged and reported unmatched; the others stay exact."""
    q = synth.mpi_endpoints(77, n_ep=3, depth_r=2500, n_src=20, n_tag=5, ragged=False, p_unmatched=0.1)
    big = synth.mpi_endpoints(78, n_ep=1, depth_r=2900, n_src=20, n_tag=5)
    # endpoint 1 gets 2900 receives: over a 2600 capacity
    eps = [q.endpoint(0), big.endpoint(0), q.endpoint(2)]
    ro = np.cumsum([0] + [len(r) for r, _ in eps])
    mo = np.cumsum([0] + [len(m) for _, m in eps])
    rh = np.concatenate([r for r, _ in eps])
    mh = np.concatenate([m[:2500] for _, m in eps])
    mo = np.cumsum([0] + [min(len(m), 2500) for _, m in eps])
    g, st = gpu_batches(MPI, 3, 2600, 2600, [(rh, None, ro, mh, None, mo)], out_cap=int(ro[-1]))
    assert st["error"] != 0 and st["rc"] == 3
    grc, gmc, _ = g[0]
    assert np.all(gmc[ro[1]:ro[2]] == -1)
    for e in (0, 2):
        sub = synth.Queues(eps[e][0], [0, len(eps[e][0])], eps[e][1][:2500], [0, min(len(eps[e][1]), 2500)])
        o, _ = oracle_batches(MPI, 1, single_batch(sub))
        assert np.array_equal(gmc[ro[e]:ro[e + 1]], remap(o[0][1], mo[e]))


def remap(omc, base):
    """Oracle message cookies of a single-endpoint run -> the multi-endpoint
    engine's (the engine numbers messages over all endpoints)."""
    return np.where(omc >= 0, omc + base, omc)


@pytest.mark.parametrize("case", ["worst", "mixed"])
def test_mpi_maximum_capacity(case):
    """Queues at the MPI level's maximum capacity (MM_MPI_MAX_MSGS, global
    workspace variant): one endpoint 24576 deep, and 3 endpoints with mixed
    wildcard types, two communicators and unexpected messages."""
    from paper_conf_ipps_klenkfed17_b200._lib import MM_MPI_MAX_MSGS
    cap = MM_MPI_MAX_MSGS
    if case == "worst":
        q = synth.worst_chain(seed=8, depth=cap, n_src=24, n_tag=6, lead_frac=0.1)
        n_ep = 1
    else:
        q = synth.mpi_endpoints(9, n_ep=3, depth_r=cap, n_src=20, n_tag=8, p_any_src=0.02, p_any_tag=0.02,
                                n_comm=2, ragged=False, p_unmatched=0.2)
        n_ep = 3
    g, qs = gpu_batches(MPI, n_ep, cap, cap, single_batch(q))
    o, _ = oracle_batches(MPI, n_ep, single_batch(q))
    assert_exact(g, o)
    assert qs["error"] == 0


@pytest.mark.parametrize("case", [
    dict(seed=1, depth=4096, lead=1024, kind="src"),
    dict(seed=2, depth=4096, lead=1000, kind="tag", n_src=40, n_tag=3),
    dict(seed=3, depth=3000, lead=2500, kind="src", msg_frac=0.5),   # groups run dry inside the run
    dict(seed=4, depth=2048, lead=37, kind="src", p_wild_after=0.3),
    dict(seed=5, depth=2048, lead=700, kind="tag", n_src=3, n_tag=50, p_wild_after=0.2),
    dict(seed=6, depth=5000, lead=5000, kind="src", n_tag=2),         # receives are all wildcards
], ids=lambda c: "s%d" % c["seed"])
def test_mpi_leading_wildcard_runs(case):
    """Wildcard runs ahead of every exact receive of their group, on the
    1024-thread deep-endpoint kernel (leading-run merge, then the chains)."""
    c = dict(case)
    q = synth.lead_runs(c.pop("seed"), **c)
    cap = int(max(np.diff(q.recv_off).max(), np.diff(q.msg_off).max(), 1))
    g, qs = gpu_batches(MPI, q.n_endpoints, cap, cap, single_batch(q))
    o, _ = oracle_batches(MPI, q.n_endpoints, single_batch(q))
    assert_exact(g, o)
    assert qs["error"] == 0


@pytest.mark.parametrize("seed", range(3))
def test_mpi_leading_runs_many_endpoints_multibatch(seed):
    """Leading runs on the 256-thread global-workspace kernel (more endpoints
    than SMs, queues too deep for shared memory), over 3 batches with
    residual queues (a residual UMQ ahead of the new messages)."""
    rng = np.random.default_rng(seed)
    q = synth.lead_runs(seed + 20, n_ep=160, depth=2048, lead=300, kind="src" if seed % 2 else "tag",
                        msg_frac=0.8, ragged=True, n_src=10, n_tag=6)
    batches = split_batches(q, 3, rng)
    g, qs = gpu_batches(MPI, q.n_endpoints, 2048, 2048, batches)
    o, oe = oracle_batches(MPI, q.n_endpoints, batches)
    assert_exact(g, o)
    rr, rm = oe.residual_depths()
    assert qs["resid_recv"] == sum(rr) and qs["resid_msg"] == sum(rm)


@pytest.mark.slow
@KERNELS
def test_mpi_config1_full(kern):
    q = synth.proxy_endpoints()
    g, qs = gpu_batches(MPI, q.n_endpoints, 1024, 1024, single_batch(q), mpi_kernel=kern)
    mr, _ = oracle.mpi_endpoints(q)
    grc, gmc, cnt = g[0]
    assert np.array_equal(grc, np.arange(len(q.recv_hdr)))
    assert np.array_equal(gmc, mr), "mismatches: %d" % int((gmc != mr).sum())
    assert int(cnt[1]) == int((mr >= 0).sum())


# ------------------------------------------------------------- relaxations


@pytest.mark.parametrize("seed", range(5))
@pytest.mark.parametrize("n", [1, 100, 4095, 4097, 50000])
@FLAT
def test_ordered_random(seed, n, flat):
    q = synth.nowild_pairs(seed, n=n, n_src=max(2, n // 50), n_tag=3, p_unmatched=0.2)
    g, _ = gpu_batches(ORD, 1, n, n, single_batch(q), flat_kernel=flat)
    o, _ = oracle_batches(ORD, 1, single_batch(q))
    assert_same_pairs(g, o)


@FLAT
def test_ordered_wide_keys_and_wildcard_values(flat):
    rng = np.random.default_rng(1)
    n = 20000
    src = rng.integers(0, 1 << 32, n, dtype=np.uint64)
    tag = rng.integers(0, 1 << 16, n, dtype=np.uint64)
    comm = rng.integers(0, 1 << 16, n, dtype=np.uint64)
    src[::7] = synth.ANY_SOURCE
    tag[::5] = synth.ANY_TAG
    rh = synth.pack(src, tag, comm)
    rh[::3] = rh[0]
    mh = rh[rng.permutation(n)]
    b = [(rh, None, np.array([0, n]), mh, None, np.array([0, n]))]
    g, _ = gpu_batches(ORD, 1, n, n, b, flat_kernel=flat)
    o, _ = oracle_batches(ORD, 1, b)
    assert_same_pairs(g, o)


@pytest.mark.parametrize("seed", range(3))
@pytest.mark.parametrize("host", [False, True], ids=["dev", "host"])
@FLAT
def test_ordered_multibatch(seed, flat, host):
    """Three batches with residual queues.  Device buffers: the bucketed
    batches' tails are decided on the device (no read-back; the next batch
    reads the residual sizes first); host buffers: the pair count comes back
    with the outputs."""
    rng = np.random.default_rng(seed)
    q = synth.nowild_pairs(seed + 3, n=30000, n_src=300, n_tag=4, p_unmatched=0.3)
    batches = split_batches(q, 3, rng)
    g, _ = gpu_batches(ORD, 1, 60000, 60000, batches, flat_kernel=flat, host=host)
    o, _ = oracle_batches(ORD, 1, batches)
    assert_same_pairs(g, o)


@FLAT
def test_ordered_all_same_key(flat):
    n = 10000
    rh = synth.pack(np.full(n, 4), np.full(n, 2))
    mh = synth.pack(np.full(n - 17, 4), np.full(n - 17, 2))
    b = [(rh, None, np.array([0, n]), mh, None, np.array([0, n - 17]))]
    g, qs = gpu_batches(ORD, 1, n, n, b, flat_kernel=flat)
    o, _ = oracle_batches(ORD, 1, b)
    assert_same_pairs(g, o)
    assert flat != 0 or qs["fallbacks"] == 1  # the bucketed run overflowed: global fallback


@pytest.mark.parametrize("sem", [ORD, UNO], ids=["ordered", "unordered"])
def test_nowild_batches_back_to_back(sem):
    """Device buffers, batches enqueued back to back with no synchronisation
    in between (the previous tail's pair count may still be in flight when the
    next batch is sized): per batch identical to the oracle (ordered) / valid
    and maximal (unordered), residual depths exact at the end."""
    import torch
    from _util import to_dev
    from paper_conf_ipps_klenkfed17_b200 import Engine
    rng = np.random.default_rng(9)
    q = synth.nowild_pairs(21, n=60000, n_src=500, n_tag=4, p_unmatched=0.3)
    batches = split_batches(q, 5, rng)
    eng = Engine(sem, 1, 120000, 120000)
    outs = []
    for (rh, rc, ro, mh, mc, mo) in batches:
        eng.post_recvs(to_dev(rh), to_dev(rc), to_dev(ro))
        eng.push_msgs(to_dev(mh), to_dev(mc), to_dev(mo))
        orc = torch.full((120000,), -7, dtype=torch.int64, device="cuda")
        omc = torch.full((120000,), -7, dtype=torch.int64, device="cuda")
        cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
        eng.match_batch(orc, omc, cnt)
        outs.append((orc, omc, cnt))
    torch.cuda.synchronize()
    g = []
    for orc, omc, cnt in outs:
        c = cnt.cpu().numpy()
        g.append((orc[: c[0]].cpu().numpy(), omc[: c[0]].cpu().numpy(), c))
    qs = eng.query()
    eng.close()
    if sem == ORD:
        o, oe = oracle_batches(ORD, 1, batches)
        assert_same_pairs(g, o)
        rr, rm = oe.residual_depths()
        assert qs["resid_recv"] == sum(rr) and qs["resid_msg"] == sum(rm)
    else:
        check_unordered_per_batch(g, batches, q.recv_hdr, q.msg_hdr)


@pytest.mark.parametrize("sem", [ORD, UNO], ids=["ordered", "unordered"])
@pytest.mark.parametrize("host", [False, True], ids=["dev", "host"])
def test_bucket_fallback_between_bucketed_batches(sem, host):
    """Batch 1 overflows the buckets (one tuple repeated thousands of times:
    the global fallback and its compaction run inside the device-decided
    tail), batch 2 is bucketed again on the residual queues of batch 1,
    batch 3 overflows again: per batch identical to the oracle (ordered) /
    valid and maximal (unordered)."""
    rng = np.random.default_rng(4)
    seq = [0, 0]  # cookies: global receive / message ids

    def batch(n, hot):
        src = rng.integers(0, 1 << 20, n)
        tag = rng.integers(0, 8, n)
        if hot:
            src[: n // 2] = 5
            tag[: n // 2] = 1
        rh = synth.pack(src, tag)
        mh = rh[rng.permutation(n)][: n - 13]
        rc = np.arange(seq[0], seq[0] + n, dtype=np.int64)
        mc = np.arange(seq[1], seq[1] + n - 13, dtype=np.int64)
        seq[0] += n
        seq[1] += n - 13
        return (rh, rc, np.array([0, n]), mh, mc, np.array([0, n - 13]))
    b = [batch(9000, True), batch(7000, False), batch(8000, True)]
    g, qs = gpu_batches(sem, 1, 30000, 30000, b, flat_kernel=0, host=host)
    assert qs["fallbacks"] == 2
    if sem == ORD:
        o, _ = oracle_batches(ORD, 1, b)
        assert_same_pairs(g, o)
    else:
        rh = np.concatenate([x[0] for x in b])
        mh = np.concatenate([x[3] for x in b])
        check_unordered_per_batch(g, b, rh, mh)


def test_ordered_long_runs_stay_on_chip():
    """Tuples repeated hundreds of times inside one bucket are ranked on chip
    (O(1) per element, no run-length limit): bit-exact, no global fallback."""
    rng = np.random.default_rng(11)
    n = 8000
    src = rng.integers(0, 1 << 20, n)
    tag = rng.integers(0, 64, n)
    src[rng.choice(n, 200, replace=False)] = 7  # one hot tuple (7, 3), 200 deep on each side
    hot = src == 7
    tag[hot] = 3
    rh = synth.pack(src, tag)
    mh = rh[rng.permutation(n)]
    b = [(rh, None, np.array([0, n]), mh, None, np.array([0, n]))]
    g, qs = gpu_batches(ORD, 1, n, n, b, flat_kernel=0)
    o, _ = oracle_batches(ORD, 1, b)
    assert_same_pairs(g, o)
    assert qs["fallbacks"] == 0


@pytest.mark.slow
@FLAT
def test_ordered_config2_full(flat):
    q = synth.nowild_pairs()
    n = len(q.recv_hdr)
    g, _ = gpu_batches(ORD, 1, n, n, single_batch(q), flat_kernel=flat)
    mr, _ = oracle.nowild_ordered(q.recv_hdr, q.msg_hdr)
    grc, gmc, cnt = g[0]
    assert np.array_equal(np.sort(grc), np.arange(n))
    got = np.empty(n, np.int64)
    got[grc] = gmc
    assert np.array_equal(got, mr), "mismatches: %d" % int((got != mr).sum())


@pytest.mark.parametrize("seed", range(5))
@pytest.mark.parametrize("n", [1, 100, 5000, 70000])
@FLAT
def test_unordered_random(seed, n, flat):
    q = synth.nowild_pairs(seed, n=n, n_src=max(2, n // 20), n_tag=3, p_unmatched=0.2)
    g, _ = gpu_batches(UNO, 1, n, n, single_batch(q), flat_kernel=flat)
    grc, gmc, cnt = g[0]
    assert np.array_equal(np.sort(grc), np.arange(n))
    o, _ = oracle_batches(UNO, 1, single_batch(q))
    # per-tuple counts are unique: compare them with the oracle's result
    orc, omc = o[0]
    om = omc >= 0
    keys, counts = np.unique(q.recv_hdr[orc[om]], return_counts=True)
    check_unordered(q.recv_hdr, q.msg_hdr, grc, gmc, dict(zip(keys.tolist(), counts.tolist())))
    assert check_min(q) == int(cnt[1])


def check_min(q):
    return sum(per_key_min(q.recv_hdr, q.msg_hdr).values())


@pytest.mark.parametrize("deep", [40, 64, 65, 66, 300, 600])
def test_unordered_deep_tuple_stays_on_chip(deep):
    """NOWILD_UNORDERED, stack kernel (k_bucket_pop): a tuple with hundreds
    of receives in one bucket (a walk of its message stack per receive would
    be quadratic) has its stack laid out flat once and its deep receives
    index it -- valid, every message expected is matched, no fallback."""
    rng = np.random.default_rng(12 + deep)
    for want in [0]:
        n = 20000
        src = rng.integers(0, 1 << 20, n)
        tag = rng.integers(0, 64, n)
        hot = rng.choice(n, deep, replace=False)
        src[hot] = 9
        tag[hot] = 4
        rh = synth.pack(src, tag)
        mh = rh[rng.permutation(n)]
        lost = np.nonzero(mh == rh[hot[0]])[0][:7]  # the hot tuple runs 7 messages short
        mh[lost] = synth.pack(rng.integers(1 << 21, 1 << 22, len(lost)), np.full(len(lost), 4))
        b = [(rh, None, np.array([0, n]), mh, None, np.array([0, n]))]
        g, qs = gpu_batches(UNO, 1, n, n, b, flat_kernel=0)
        grc, gmc, cnt = g[0]
        assert np.array_equal(np.sort(grc), np.arange(n))
        m = gmc >= 0
        assert np.array_equal(rh[grc[m]], mh[gmc[m]]) and len(np.unique(gmc[m])) == int(m.sum())
        assert int(m.sum()) == sum(per_key_min(rh, mh).values())  # maximal per tuple
        assert qs["fallbacks"] == want


@pytest.mark.parametrize("seed", range(3))
@pytest.mark.parametrize("host", [False, True], ids=["dev", "host"])
@FLAT
def test_unordered_multibatch(seed, flat, host):
    rng = np.random.default_rng(seed)
    q = synth.nowild_pairs(seed + 7, n=20000, n_src=200, n_tag=3, p_unmatched=0.3)
    batches = split_batches(q, 3, rng)
    g, _ = gpu_batches(UNO, 1, 40000, 40000, batches, flat_kernel=flat, host=host)
    # across all batches: every pair has equal tuples, every element used once,
    # and the total per tuple is min(#recv, #msg) of the whole input
    rc = np.concatenate([x[0] for x in g])
    mc = np.concatenate([x[1] for x in g])
    m = mc >= 0
    assert len(np.unique(rc[m])) == m.sum() and len(np.unique(mc[m])) == m.sum()
    assert np.array_equal(q.recv_hdr[rc[m]], q.msg_hdr[mc[m]])
    assert int(m.sum()) == check_min(q)
    check_unordered_per_batch(g, batches, q.recv_hdr, q.msg_hdr)


@pytest.mark.slow
@FLAT
def test_unordered_config3_per_gpu(flat):
    q = synth.nowild_pairs(3, n=1 << 25, n_src=1 << 20, n_tag=1 << 12)
    n = len(q.recv_hdr)
    g, _ = gpu_batches(UNO, 1, n, n, single_batch(q), flat_kernel=flat)
    grc, gmc, cnt = g[0]
    m = gmc >= 0
    assert np.array_equal(q.recv_hdr[grc[m]], q.msg_hdr[gmc[m]])
    assert len(np.unique(gmc[m])) == int(m.sum())
    keys, mins = per_key_min_np(q.recv_hdr, q.msg_hdr)
    assert int(m.sum()) == int(mins.sum()) == int(cnt[1])


@pytest.mark.slow
def test_unordered_config3_full_256m():
    """configs[3] at its named size on one B200: 256M receive/message pairs
    in one engine (§VI.C l.213-221; the 8-GPU run shards the same key
    space).  Checked on the device with torch (the properties reading R6
    fixes at any size): every receive reported once, matched pairs carry
    equal tuples, each message used once, and the match count equals
    sum over tuples of min(#recv, #msg) -- with validity this forces every
    tuple to its own min (a maximal pairing)."""
    import torch
    from paper_conf_ipps_klenkfed17_b200 import MM_SEM_NOWILD_UNORDERED, Engine
    n = 1 << 28
    q = synth.nowild_pairs(3, n=n, n_src=1 << 20, n_tag=1 << 12)
    rh = torch.from_numpy(q.recv_hdr.view(np.int64)).cuda()
    mh = torch.from_numpy(q.msg_hdr.view(np.int64)).cuda()
    del q
    eng = Engine(MM_SEM_NOWILD_UNORDERED, 1, n, n)
    orc = torch.empty(n, dtype=torch.int64, device="cuda")
    omc = torch.empty(n, dtype=torch.int64, device="cuda")
    cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
    eng.post_recvs(rh)
    eng.push_msgs(mh)
    eng.match_batch(orc, omc, cnt)
    st = eng.query()
    eng.close()
    assert st["error"] == 0
    assert int(cnt[0]) == n
    assert torch.equal(torch.sort(orc).values, torch.arange(n, device="cuda"))
    m = omc >= 0
    n_matched = int(m.sum())
    assert n_matched == int(cnt[1])
    assert torch.equal(rh[orc[m]], mh[omc[m]]), "matched tuples differ"
    used = torch.sort(omc[m]).values
    assert not bool((used[1:] == used[:-1]).any()), "a message matched twice"
    del used, orc, omc, m
    kr, cr = torch.unique_consecutive(torch.sort(rh).values, return_counts=True)
    km, cm = torch.unique_consecutive(torch.sort(mh).values, return_counts=True)
    pos = torch.searchsorted(km, kr).clamp(max=len(km) - 1)
    hit = km[pos] == kr
    assert n_matched == int(torch.minimum(cr[hit], cm[pos[hit]]).sum())


# ------------------------------------------------------------------- route


@pytest.mark.parametrize("world,by", [(1, 0), (2, 0), (8, 0), (5, 1), (256, 0)])
def test_route_stable_partition(world, by):
    import torch
    from paper_conf_ipps_klenkfed17_b200 import route
    rng = np.random.default_rng(world)
    n = 30011
    if by == 0:
        a = synth.pack(rng.integers(0, 1000, n), rng.integers(0, 50, n))
        h = np.array([oracle.jenkins32((int(x) & 0xFFFFFFFF) ^ oracle.jenkins32(int(x) >> 32)) for x in a],
                     dtype=np.uint64)
        owner = (h * np.uint64(world)) >> np.uint64(32)
    else:
        owner = rng.integers(0, world, n).astype(np.uint64)
        a = (owner << np.uint64(40)) | rng.integers(0, 1 << 40, n).astype(np.uint64)
    b = rng.integers(0, 1 << 60, n)
    da = torch.from_numpy(a.view(np.int64)).cuda()
    db = torch.from_numpy(b).cuda()
    oa = torch.empty_like(da)
    ob = torch.empty_like(db)
    counts = np.zeros(world, np.int64)
    route(da, db, world, by, oa, ob, counts)
    # b == NULL: generated cookies cookie_base + k
    oa2, ob2 = torch.empty_like(da), torch.empty_like(db)
    route(da, None, world, by, oa2, ob2, counts, cookie_base=(3 << 40) + 7)
    assert np.array_equal(ob2.cpu().numpy(), (3 << 40) + 7 + np.argsort(owner, kind="stable"))
    order = np.argsort(owner, kind="stable")
    assert np.array_equal(counts, np.bincount(owner.astype(np.int64), minlength=world))
    assert np.array_equal(oa.cpu().numpy().view(np.uint64), a[order])
    assert np.array_equal(ob.cpu().numpy(), b[order])
