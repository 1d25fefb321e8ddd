"""Host logic of the multi-GPU path over gloo, world_size 2 (CPU).

The CUDA kernels are replaced by a CPU stand-in (route: the same owner rule
written with the oracle's Jenkins hash; engine: the oracle's batch engine), so
what is tested is parallel.py's orchestration: owner partition, count
exchange, split bookkeeping, global order (origin rank, local index) at the
owner, and the return trip of results.  The sharded result must equal the
oracle run on the concatenation of all ranks' inputs.
"""
import os
import subprocess
import sys

import pytest

from conftest import ROOT

WORKER = r'''
import os, sys, json
sys.path.insert(0, os.environ["ROOT"])
import numpy as np, torch, torch.distributed as dist
import oracle, synth
from paper_conf_ipps_klenkfed17_b200.parallel import ShardedMatcher, split_endpoints

SHIFT = 40

class CpuOps:
    def route(self, a, b, world, by, base):
        a_np = a.numpy().view(np.uint64)
        n = len(a_np)
        if by == 0:
            h = np.array([oracle.jenkins32((int(x) & 0xFFFFFFFF) ^ oracle.jenkins32(int(x) >> 32)) for x in a_np],
                         dtype=np.uint64)
            owner = ((h * np.uint64(world)) >> np.uint64(32)).astype(np.int64)
        else:
            owner = (a_np >> np.uint64(SHIFT)).astype(np.int64)
        bb = b.numpy() if b is not None else np.int64(base) + np.arange(n, dtype=np.int64)
        nb = world
        if by == 2:  # matched before unmatched within each origin
            owner = 2 * owner + (bb == -1)
            nb = 2 * world
        order = np.argsort(owner, kind="stable")
        return (torch.from_numpy(a_np[order].view(np.int64).copy()), torch.from_numpy(bb[order].copy()),
                torch.from_numpy(np.bincount(owner, minlength=nb).astype(np.int64)))

    def make_engine(self, sem, cap):
        return OracleAsEngine(sem)

    def empty(self, n, like):
        return torch.empty(n, dtype=torch.int64)

    def zeros(self, n, like):
        return torch.zeros(n, dtype=torch.int64)

class OracleAsEngine:
    def __init__(self, sem):
        self.e = oracle.OracleEngine(sem, 1)
    def post_recvs(self, h, c):
        self.e.post_recvs(h.numpy().view(np.uint64), c.numpy())
    def push_msgs(self, h, c):
        self.e.push_msgs(h.numpy().view(np.uint64), c.numpy())
    def match_batch(self, orc, omc, cnt):
        rc, mc = self.e.match_batch()
        n = len(rc)
        orc[:n] = torch.from_numpy(rc); omc[:n] = torch.from_numpy(mc)
        cnt[0] = n; cnt[1] = int((mc >= 0).sum())
    def close(self):
        pass

dist.init_process_group("gloo")
rank, world = dist.get_rank(), dist.get_world_size()
sem = int(os.environ["SEM"])
cuda = os.environ.get("OPS") == "cuda"  # the real kernels (mm_route + Engine) on the one GPU
N, NB = int(os.environ.get("N", "300")), int(os.environ.get("NB", "2"))
res = {"lo_hi": split_endpoints(10, world, rank)}
outs = []
if cuda:
    torch.cuda.set_device(0)
    from paper_conf_ipps_klenkfed17_b200.parallel import CudaOps
    ops = CudaOps()
else:
    ops = CpuOps()
m = ShardedMatcher(sem, capacity=8 * N * world, ops=ops)
for b in range(NB):
    q = synth.nowild_pairs(100 * b + rank, n=N, n_src=max(12, N // 25), n_tag=3, p_unmatched=0.25)
    rh = torch.from_numpy(q.recv_hdr.view(np.int64).copy())
    mh = torch.from_numpy(q.msg_hdr.view(np.int64).copy())
    if cuda:
        rh, mh = rh.cuda(), mh.cuda()
    rc, mc = m.match(rh, mh)
    if cuda:
        torch.cuda.synchronize()
        rc, mc = rc.cpu(), mc.cpu()
    outs.append((rc.numpy().tolist(), mc.numpy().tolist()))
res["outs"] = outs
res["host_syncs"] = m.host_syncs
m.close()
with open(os.path.join(os.environ["OUTDIR"], "rank%d.json" % rank), "w") as f:
    json.dump(res, f)
dist.destroy_process_group()
'''


def run_world2(tmp_path, sem, ops="cpu", n=300, nb=2):
    script = tmp_path / "worker.py"
    script.write_text(WORKER)
    env = dict(os.environ, ROOT=ROOT, OUTDIR=str(tmp_path), SEM=str(sem), OPS=ops, N=str(n), NB=str(nb))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nproc-per-node", "2", "--master-addr", "127.0.0.1",
           "--master-port", str(29500 + (os.getpid() % 1000)), str(script)]
    p = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=600)
    assert p.returncode == 0, p.stderr[-3000:]
    import json
    return [json.load(open(tmp_path / ("rank%d.json" % r))) for r in range(2)]


def global_reference(sem, world=2, n=300, nb=2):
    """The oracle on the concatenation of all ranks' inputs, batch by batch,
    cookies (origin << 40) | local index."""
    import numpy as np

    import oracle
    import synth
    eng = oracle.OracleEngine(sem, 1)
    res = []
    seq = {("r", r): 0 for r in range(world)}
    seq.update({("m", r): 0 for r in range(world)})
    for b in range(nb):
        qs = [synth.nowild_pairs(100 * b + r, n=n, n_src=max(12, n // 25), n_tag=3, p_unmatched=0.25)
              for r in range(world)]
        rh = np.concatenate([q.recv_hdr for q in qs])
        mh = np.concatenate([q.msg_hdr for q in qs])
        def ck(side, attr):
            out = []
            for r, q in enumerate(qs):
                n = len(getattr(q, attr))
                out.append((np.int64(r) << 40) + seq[(side, r)] + np.arange(n, dtype=np.int64))
                seq[(side, r)] += n
            return np.concatenate(out)
        eng.post_recvs(rh, ck("r", "recv_hdr"))
        eng.push_msgs(mh, ck("m", "msg_hdr"))
        res.append(eng.match_batch())
    return res


def global_inputs(n, nb, world=2):
    """Per batch: {recv cookie: header}, {msg cookie: header} over all ranks
    (cookie = (origin << 40) | running local index)."""
    import synth
    seq, out = {}, []
    for b in range(nb):
        hr, hm = {}, {}
        for r in range(world):
            q = synth.nowild_pairs(100 * b + r, n=n, n_src=max(12, n // 25), n_tag=3, p_unmatched=0.25)
            for side, arr, d in (("r", q.recv_hdr, hr), ("m", q.msg_hdr, hm)):
                s0 = seq.get((side, r), 0)
                for i, h in enumerate(arr.tolist()):
                    d[(r << 40) + s0 + i] = h
                seq[(side, r)] = s0 + len(arr)
        out.append((hr, hm))
    return out


def check_unordered_batches(ranks, inputs):
    """NOWILD_UNORDERED over several batches (reading R6, per batch): the
    snapshot is our own residual plus the batch; matched pairs have equal
    tuples and use each snapshot message once; every tuple gets
    min(#recv, #msg) of the snapshot (maximal); the residuals carry over."""
    from collections import Counter
    res_r, res_m = {}, {}
    for b, (hr, hm) in enumerate(inputs):
        snap_r = {**res_r, **hr}
        snap_m = {**res_m, **hm}
        got = {}
        for r in range(2):
            rc, mc = ranks[r]["outs"][b]
            for x, y in zip(rc, mc):
                assert (x >> 40) == r, "a result came back to the wrong origin"
                assert x not in got, "a receive reported twice"
                got[x] = y
        assert set(got) == set(snap_r), "batch %d: snapshot receives differ from residual + batch" % b
        used = set()
        per = Counter()
        for x, y in got.items():
            if y >= 0:
                assert y in snap_m and y not in used, "a message matched twice or not in the snapshot"
                assert snap_r[x] == snap_m[y], "unequal tuples matched"
                used.add(y)
                per[snap_r[x]] += 1
        cr, cm = Counter(snap_r.values()), Counter(snap_m.values())
        want = {k: min(v, cm[k]) for k, v in cr.items() if min(v, cm[k]) > 0}
        assert dict(per) == want, "batch %d: not a maximal pairing per tuple" % b
        res_r = {x: snap_r[x] for x, y in got.items() if y < 0}
        res_m = {y: h for y, h in snap_m.items() if y not in used}


def check_world2(ranks, ref, sem, nb, n=300):
    if sem == 1:
        for b in range(nb):
            got = {}
            for r in range(2):
                rc, mc = ranks[r]["outs"][b]
                for x, y in zip(rc, mc):
                    assert (x >> 40) == r, "a result came back to the wrong origin"
                    assert x not in got, "a receive reported twice"
                    got[x] = y
            orc, omc = ref[b]
            assert got == dict(zip(orc.tolist(), omc.tolist()))  # ordered: bit-exact with the global oracle
    else:
        check_unordered_batches(ranks, global_inputs(n, nb))
    for r in range(2):
        assert ranks[r]["host_syncs"] == nb, "one host read-back per batch"


@pytest.mark.parametrize("sem", [1, 2])
def test_sharded_matcher_world2(tmp_path, sem):
    ranks = run_world2(tmp_path, sem)
    assert ranks[0]["lo_hi"] == [0, 5] and ranks[1]["lo_hi"] == [5, 10]
    check_world2(ranks, global_reference(sem), sem, 2)


@pytest.mark.gpu
@pytest.mark.parametrize("sem", [1, 2])
def test_sharded_matcher_world2_cuda(tmp_path, sem):
    """The real multi-GPU path -- ShardedMatcher over CudaOps: mm_route on the
    device, the Engine's kernels at each owner, the return route by origin
    (by=2) -- two ranks sharing the one GPU over gloo, 3 batches with
    residual queues, against the oracle on the concatenated input."""
    n, nb = 20000, 3
    ranks = run_world2(tmp_path, sem, ops="cuda", n=n, nb=nb)
    check_world2(ranks, global_reference(sem, n=n, nb=nb) if sem == 1 else None, sem, nb, n=n)
