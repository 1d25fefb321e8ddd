#!/usr/bin/env python
"""Host-side time of each API call of one bench level step (diagnostic)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, bench
import paper_conf_ipps_klenkfed17_b200 as mm
level = sys.argv[1] if len(sys.argv) > 1 else "unordered"
q = bench.ordered_workload(0, 1) if level == "ordered" else bench.unordered_workload(0)
n = len(q.recv_hdr)
sem = mm.MM_SEM_NOWILD_ORDERED if level == "ordered" else mm.MM_SEM_NOWILD_UNORDERED
eng = mm.Engine(sem, 1, n, n)
rh, mh = bench.to_dev(q.recv_hdr), bench.to_dev(q.msg_hdr)
orc = torch.empty(n, dtype=torch.int64, device="cuda"); omc = torch.empty_like(orc)
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
tt = {}
for it in range(8):
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter(); e0.record()
    eng.reset(); t1 = time.perf_counter()
    eng.post_recvs(rh); t2 = time.perf_counter()
    eng.push_msgs(mh); t3 = time.perf_counter()
    eng.match_batch(orc, omc, cnt); t4 = time.perf_counter()
    e1.record(); torch.cuda.synchronize(); t5 = time.perf_counter()
    if it >= 3:
        for k, v in (("reset", t1 - t0), ("post", t2 - t1), ("push", t3 - t2), ("match(host)", t4 - t3), ("drain", t5 - t4), ("wall", t5 - t0)):
            tt.setdefault(k, []).append(v * 1e6)
        tt.setdefault("events", []).append(e0.elapsed_time(e1) * 1e3)
for k, v in tt.items():
    print("%-12s %8.1f us" % (k, sum(v) / len(v)))
q1 = eng.query(); print("kernel_ns/run %.1f us" % (q1["kernel_ns"] / max(1, q1["kernel_runs"]) / 1e3))
