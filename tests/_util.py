"""Helpers shared by the parity tests: drive the CUDA path and the oracle on
the same seeded synth.Queues and compare."""
from collections import Counter

import numpy as np

import oracle


def to_dev(a):
    import torch
    if a is None:
        return None
    a = np.ascontiguousarray(a)
    if a.dtype == np.uint64:
        a = a.view(np.int64)
    return torch.from_numpy(a.copy()).cuda()


def gpu_batches(sem, n_ep, rcap, mcap, batches, host=False, out_cap=None, mpi_kernel=None, flat_kernel=None,
                pipeline=None):
    """batches: list of (recv_hdr, recv_cookie, recv_off, msg_hdr, msg_cookie, msg_off).
    host: False (device buffers), True (host inputs and outputs), "in" (host
    inputs, device outputs), "out" (device inputs, host outputs), "pinned"
    (page-locked host inputs and outputs) or "pinned-mapped" (the same with
    MM_HOST_OUT_MAPPED: the MPI level writes the outputs in place through
    their mapped addresses).
    pipeline: MM_OPT_PIPELINE_CHUNKS value (None = engine default).
    Returns a list of (out_rc, out_mc) numpy arrays, one per batch."""
    import torch
    from paper_conf_ipps_klenkfed17_b200 import Engine
    from paper_conf_ipps_klenkfed17_b200._lib import MM_OPT_PIPELINE_CHUNKS
    eng = Engine(sem, n_ep, rcap, mcap, mpi_kernel=mpi_kernel, flat_kernel=flat_kernel)
    if pipeline is not None:
        eng.set_option(MM_OPT_PIPELINE_CHUNKS, pipeline)
    pinned = host in ("pinned", "pinned-mapped")
    if host == "pinned-mapped":
        from paper_conf_ipps_klenkfed17_b200._lib import MM_HOST_OUT_MAPPED, MM_OPT_HOST_OUT
        eng.set_option(MM_OPT_HOST_OUT, MM_HOST_OUT_MAPPED)
    host_in = host is True or host == "in" or pinned
    host_out = host is True or host == "out" or pinned

    def hbuf(a, dtype=np.int64):  # pageable numpy, or a page-locked numpy view
        if a is None:
            return None
        a = np.ascontiguousarray(a, dtype)
        if not pinned:
            return a
        t = torch.empty(a.shape, dtype=torch.int64).pin_memory()
        t.numpy().view(dtype)[:] = a
        keep.append(t)
        return t.numpy().view(dtype)

    keep = []  # page-locked buffers stay alive until the engine is closed
    res = []
    for (rh, rc, ro, mh, mc, mo) in batches:
        if host_in:
            eng.post_recvs(hbuf(rh, np.uint64), hbuf(rc), hbuf(ro))
            eng.push_msgs(hbuf(mh, np.uint64), hbuf(mc), hbuf(mo))
        else:
            eng.post_recvs(to_dev(rh), to_dev(rc), to_dev(ro))
            eng.push_msgs(to_dev(mh), to_dev(mc), to_dev(mo))
        cap = out_cap if out_cap is not None else n_ep * rcap
        if host_out:
            orc = hbuf(np.full(cap, -7, np.int64))
            omc = hbuf(np.full(cap, -7, np.int64))
            cnt = hbuf(np.zeros(2, np.int64))
            eng.match_batch(orc, omc, cnt)
            n = min(int(cnt[0]), cap)
            res.append((orc[:n].copy(), omc[:n].copy(), cnt.copy()))
        else:
            orc = torch.full((cap,), -7, dtype=torch.int64, device="cuda")
            omc = torch.full((cap,), -7, dtype=torch.int64, device="cuda")
            cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
            eng.match_batch(orc, omc, cnt)
            torch.cuda.synchronize()
            c = cnt.cpu().numpy()
            n = min(int(c[0]), cap)
            res.append((orc[:n].cpu().numpy(), omc[:n].cpu().numpy(), c))
    q = eng.query(raise_on_error=False)
    eng.close()
    return res, q


def oracle_batches(sem, n_ep, batches):
    eng = oracle.OracleEngine(sem, n_ep)
    res = []
    for (rh, rc, ro, mh, mc, mo) in batches:
        eng.post_recvs(rh, rc, ro)
        eng.push_msgs(mh, mc, mo)
        res.append(eng.match_batch())
    return res, eng


def single_batch(q):
    return [(q.recv_hdr, None, q.recv_off, q.msg_hdr, None, q.msg_off)]


def split_batches(q, k, rng):
    """Split every endpoint's queues into k consecutive pieces at random cuts."""
    out = []
    cuts_r = [np.sort(rng.integers(q.recv_off[e], q.recv_off[e + 1] + 1, k - 1)) for e in range(q.n_endpoints)]
    cuts_m = [np.sort(rng.integers(q.msg_off[e], q.msg_off[e + 1] + 1, k - 1)) for e in range(q.n_endpoints)]
    for b in range(k):
        def piece(off, cuts, hdr):
            hs, cs, o = [], [], [0]
            for e in range(q.n_endpoints):
                bounds = [off[e], *cuts[e], off[e + 1]]
                lo, hi = int(bounds[b]), int(bounds[b + 1])
                hs.append(hdr[lo:hi]); cs.append(np.arange(lo, hi, dtype=np.int64)); o.append(o[-1] + hi - lo)
            return np.concatenate(hs).astype(np.uint64), np.concatenate(cs), np.array(o, np.int64)
        rh, rc, ro = piece(q.recv_off, cuts_r, q.recv_hdr)
        mh, mc, mo = piece(q.msg_off, cuts_m, q.msg_hdr)
        out.append((rh, rc, ro, mh, mc, mo))
    return out


def check_unordered(recv_hdr_by_cookie, msg_hdr_by_cookie, out_rc, out_mc, expect_per_key=None):
    """Validity of an unordered result: matched pairs have equal tuples, each
    message used at most once, and (if given) per-tuple match counts equal."""
    m = out_mc >= 0
    rk = recv_hdr_by_cookie[out_rc[m]]
    mk = msg_hdr_by_cookie[out_mc[m]]
    assert np.array_equal(rk, mk), "matched tuples differ"
    assert len(np.unique(out_mc[m])) == int(m.sum()), "a message matched twice"
    if expect_per_key is not None:
        keys, cnt = np.unique(rk, return_counts=True)
        got = dict(zip(keys.tolist(), cnt.tolist()))
        assert got == expect_per_key


def per_key_min(recv_hdr, msg_hdr):
    cr = Counter(recv_hdr.tolist())
    cm = Counter(msg_hdr.tolist())
    out = {}
    for k in cr:
        v = min(cr[k], cm.get(k, 0))
        if v:
            out[k] = v
    return out


def per_key_min_np(recv_hdr, msg_hdr):
    """Vectorised per-key min(#recv, #msg) as (keys, counts) arrays."""
    ku, cu = np.unique(recv_hdr, return_counts=True)
    km, cm = np.unique(msg_hdr, return_counts=True)
    common, ia, ib = np.intersect1d(ku, km, assume_unique=True, return_indices=True)
    return common, np.minimum(cu[ia], cm[ib])


def check_unordered_per_batch(results, batches, recv_hdr_by_cookie, msg_hdr_by_cookie):
    """NOWILD_UNORDERED over several batches, batch by batch (reading R6):
    the snapshot is the engine's own residual plus the batch; every snapshot
    receive is reported once; matched pairs have equal tuples and use each
    snapshot message at most once; every tuple gets min(#recv, #msg) of the
    snapshot (a maximal pairing); the residuals carry over."""
    res_r = np.zeros(0, np.int64)
    res_m = np.zeros(0, np.int64)
    for b, ((grc, gmc, _), (rh, rc, ro, mh, mc, mo)) in enumerate(zip(results, batches)):
        snap_r = np.concatenate([res_r, np.asarray(rc, np.int64)])
        snap_m = np.concatenate([res_m, np.asarray(mc, np.int64)])
        assert np.array_equal(np.sort(grc), np.sort(snap_r)), "batch %d: snapshot receives" % b
        m = gmc >= 0
        used = gmc[m]
        assert len(np.unique(used)) == len(used), "batch %d: a message matched twice" % b
        assert np.isin(used, snap_m).all(), "batch %d: a message outside the snapshot" % b
        assert np.array_equal(recv_hdr_by_cookie[grc[m]], msg_hdr_by_cookie[used]), "batch %d: tuples" % b
        keys, mins = per_key_min_np(recv_hdr_by_cookie[snap_r], msg_hdr_by_cookie[snap_m])
        got_k, got_c = np.unique(recv_hdr_by_cookie[grc[m]], return_counts=True)
        assert np.array_equal(got_k, keys) and np.array_equal(got_c, mins), "batch %d: not maximal per tuple" % b
        res_r = grc[~m]
        res_m = snap_m[~np.isin(snap_m, used)]
