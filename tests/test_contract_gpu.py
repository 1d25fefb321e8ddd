"""The C-ABI's stated contracts (include/mm.h), checked on the GPU.

* capacity overflow (mm.h header comment): the affected endpoint's batch is
  rejected -- its receives reported unmatched, its queues keep their previous
  contents, its pending elements dropped -- while every other endpoint is
  matched as the oracle says;
* host input lifetime (mm_post_recvs / mm_push_msgs): page-locked input
  buffers may be overwritten as soon as mm_match_batch returns, also with
  device outputs (no synchronising copy-back);
* mm_route by == 1 with a cookie that names no rank: memory-safe, placed after
  every owner's group, uncounted, MM_ERR_ARG with host counts.
"""
import numpy as np
import pytest

import oracle
import synth
from _util import oracle_batches, single_batch, to_dev

pytestmark = pytest.mark.gpu

MPI = oracle.SEM_MPI
KERNELS = pytest.mark.parametrize("kern", [1, 2], ids=["matrix", "fifo"])


def csr(per_ep):
    """per_ep: list over endpoints of (headers, cookies) -> (hdr, cookie, off)."""
    off = np.zeros(len(per_ep) + 1, np.int64)
    off[1:] = np.cumsum([len(h) for h, _ in per_ep])
    hdr = np.concatenate([np.asarray(h, np.uint64) for h, _ in per_ep]) if off[-1] else np.zeros(0, np.uint64)
    ck = np.concatenate([np.asarray(c, np.int64) for _, c in per_ep]) if off[-1] else np.zeros(0, np.int64)
    return hdr, ck, off


def tuples(rng, n, e):
    return synth.pack(rng.integers(0, 4, n) + 10 * e, rng.integers(0, 3, n))


@KERNELS
@pytest.mark.parametrize("where", ["kernel", "materialize"])
def test_capacity_overflow_rejects_the_endpoint_batch(kern, where):
    """Endpoint 0 overflows in batch 2 (snapshot above capacity in the
    matching kernel, or a second post that no longer fits when the first is
    moved into the queue); endpoints 1-2 do not.  Expected: endpoint 0's
    batch-2 receives are reported with MM_NO_MATCH, its queues are as after
    batch 1, and every other result equals the oracle run on the same batches
    with endpoint 0's rejected elements removed."""
    rng = np.random.default_rng(11 + kern)
    cap, n_ep = 32, 3
    ck = iter(range(10 ** 6))

    def side(n_per_ep, _tag):
        return [(tuples(rng, n, e), [next(ck) for _ in range(n)]) for e, n in enumerate(n_per_ep)]

    b1r, b1m = side([12, 10, 8], 1), side([6, 10, 4], 1)
    b3r, b3m = side([2, 3, 1], 3), side([20, 12, 9], 3)
    if where == "kernel":
        b2r = [side([30], 0)[0], *side([0, 5, 4], 2)[1:]]  # ep0: residual (>= 6) + 30 > 32
        b2m = side([3, 2, 2], 2)
        posts2 = [b2r]
        dropped = [b2r[0], b2m[0]]  # the kernel rejects both of ep0's pending sides
    else:
        first, second = side([16, 2, 1], 2), side([20, 1, 1], 2)  # ep0: resid (<= 12) + 16 + 20 > 32
        third = side([4, 1, 0], 2)
        b2m = side([0, 2, 2], 2)
        posts2 = [first, second, third]
        dropped = [second[0]]  # the second post no longer fits when it is moved into the queue

    import torch
    from paper_conf_ipps_klenkfed17_b200 import Engine
    eng = Engine(MPI, n_ep, cap, cap, mpi_kernel=kern)
    results = []
    for posts, msgs in [([b1r], b1m), (posts2, b2m), ([b3r], b3m)]:
        for p in posts:
            h, c, o = csr(p)
            eng.post_recvs(to_dev(h), to_dev(c), to_dev(o))
        h, c, o = csr(msgs)
        eng.push_msgs(to_dev(h), to_dev(c), to_dev(o))
        out = n_ep * cap * 2
        orc = torch.full((out,), -7, dtype=torch.int64, device="cuda")
        omc = torch.full((out,), -7, dtype=torch.int64, device="cuda")
        cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
        eng.match_batch(orc, omc, cnt)
        torch.cuda.synchronize()
        n = int(cnt[0])
        results.append((orc[:n].cpu().numpy(), omc[:n].cpu().numpy()))
    st = eng.query(raise_on_error=False)
    eng.close()
    assert st["error"] != 0 and st["rc"] == 3

    # oracle: the same batches with endpoint 0's rejected elements removed
    def keep(side):
        return [([], []) if (e == 0 and any(side[0] is d for d in dropped)) else side[e] for e in range(n_ep)]
    oe = oracle.OracleEngine(MPI, n_ep)
    expect = []
    for posts, msgs in [([b1r], b1m), (posts2, b2m), ([b3r], b3m)]:
        for p in posts:
            h, c, o = csr(keep(p))
            oe.post_recvs(h, c, o)
        h, c, o = csr(keep(msgs))
        oe.push_msgs(h, c, o)
        expect.append(oe.match_batch())
    # batches 1 and 3 equal the oracle exactly
    for b in (0, 2):
        assert np.array_equal(results[b][0], expect[b][0]) and np.array_equal(results[b][1], expect[b][1]), b
    grc, gmc = results[1]
    orc, omc = expect[1]
    if where == "kernel":
        r0 = int(np.sum(expect[0][1][:12] == -1))  # ep0's residual receives after batch 1
        n0 = r0 + 30
        assert np.array_equal(grc[:r0], orc[:r0]) and np.all(omc[:r0] == -1)
        assert np.array_equal(grc[r0:n0], np.asarray(b2r[0][1]))
        assert np.all(gmc[:n0] == -1)
        assert np.array_equal(grc[n0:], orc[r0:]) and np.array_equal(gmc[n0:], omc[r0:])
    else:
        assert np.array_equal(grc, orc) and np.array_equal(gmc, omc)


@KERNELS
@pytest.mark.parametrize("n_ep", [16, 300])
def test_pinned_inputs_may_be_overwritten_after_match_batch(kern, n_ep):
    """Page-locked host inputs, device outputs: the caller overwrites the
    input buffers right after mm_match_batch returns; the results must be
    those of the original inputs (n_ep = 300 takes the host-buffer pipeline)."""
    import torch
    from paper_conf_ipps_klenkfed17_b200 import Engine
    q = synth.mpi_endpoints(21, n_ep=n_ep, depth_r=256, ragged=True, p_unmatched=0.2)
    eng = Engine(MPI, n_ep, 256, 256, mpi_kernel=kern)
    pins = []
    for _ in range(3):
        rh = torch.from_numpy(q.recv_hdr.view(np.int64).copy()).pin_memory()
        ro = torch.from_numpy(q.recv_off.copy()).pin_memory()
        mh = torch.from_numpy(q.msg_hdr.view(np.int64).copy()).pin_memory()
        mo = torch.from_numpy(q.msg_off.copy()).pin_memory()
        eng.reset()
        eng.post_recvs(rh, None, ro)
        eng.push_msgs(mh, None, mo)
        n = len(q.recv_hdr)
        orc = torch.empty(n, dtype=torch.int64, device="cuda")
        omc = torch.empty(n, dtype=torch.int64, device="cuda")
        cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
        eng.match_batch(orc, omc, cnt)
        for t in (rh, mh):
            t.fill_(0x0123456789)  # the caller reuses its buffers at once
        torch.cuda.synchronize()
        pins.append((orc.cpu().numpy(), omc.cpu().numpy()))
    eng.close()
    o, _ = oracle_batches(MPI, n_ep, single_batch(q))
    for grc, gmc in pins:
        assert np.array_equal(grc, o[0][0]) and np.array_equal(gmc, o[0][1])


def test_route_cookie_naming_no_rank():
    import torch
    from paper_conf_ipps_klenkfed17_b200 import MMError, route
    rng = np.random.default_rng(5)
    world, n = 4, 5000
    owner = rng.integers(0, world, n).astype(np.uint64)
    bad = rng.random(n) < 0.01
    owner[bad] = np.uint64(world) + rng.integers(0, 1000, int(bad.sum())).astype(np.uint64)
    owner[7] = np.uint64((1 << 24) - 1)  # MM_NO_MATCH-like all-ones origin bits
    bad[7] = True
    a = (owner << np.uint64(40)) | rng.integers(0, 1 << 40, n).astype(np.uint64)
    da = torch.from_numpy(a.view(np.int64)).cuda()
    oa, ob = torch.empty_like(da), torch.empty_like(da)
    dcounts = torch.zeros(world, dtype=torch.int64, device="cuda")
    route(da, None, world, 1, oa, ob, dcounts)
    torch.cuda.synchronize()
    good = ~bad
    expect_counts = np.bincount(owner[good].astype(np.int64), minlength=world)
    assert np.array_equal(dcounts.cpu().numpy(), expect_counts)
    k = int(good.sum())
    order = np.argsort(np.where(good, owner, np.uint64(world)), kind="stable")
    assert np.array_equal(oa.cpu().numpy().view(np.uint64), a[order])
    assert np.array_equal(ob.cpu().numpy()[k:], np.nonzero(bad)[0])
    with pytest.raises(MMError):
        route(da, None, world, 1, oa, ob, np.zeros(world, np.int64))


@pytest.mark.parametrize("world", [1, 3, 8, 255])
def test_route_by_origin_matched_first(world):
    """mm_route by == 2 (the sharded return trip): grouped by origin rank,
    within each origin the matched results (b != MM_NO_MATCH) before the
    unmatched ones, each part in input order; counts {matched, unmatched}
    per origin; a cookie naming no rank after everything, uncounted."""
    import torch
    from paper_conf_ipps_klenkfed17_b200 import route
    rng = np.random.default_rng(world)
    n = 40000
    owner = rng.integers(0, world, n).astype(np.uint64)
    bad = rng.random(n) < 0.002
    owner[bad] = np.uint64(world + 3)
    a = (owner << np.uint64(40)) | rng.integers(0, 1 << 40, n).astype(np.uint64)
    b = np.where(rng.random(n) < 0.3, -1, rng.integers(0, 1 << 50, n)).astype(np.int64)
    da, db = torch.from_numpy(a.view(np.int64)).cuda(), torch.from_numpy(b).cuda()
    oa, ob = torch.empty_like(da), torch.empty_like(db)
    counts = torch.zeros(2 * world, dtype=torch.int64, device="cuda")
    route(da, db, world, 2, oa, ob, counts)
    torch.cuda.synchronize()
    key = np.where(bad, 2 * world, 2 * owner.astype(np.int64) + (b == -1))
    order = np.argsort(key, kind="stable")
    assert np.array_equal(oa.cpu().numpy().view(np.uint64), a[order])
    assert np.array_equal(ob.cpu().numpy(), b[order])
    assert np.array_equal(counts.cpu().numpy(), np.bincount(key[~bad], minlength=2 * world))
