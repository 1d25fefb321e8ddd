#!/usr/bin/env python
"""Kernel timeline of one step (start offset, duration, gap before) via torch.profiler (diagnostic)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, bench
import paper_conf_ipps_klenkfed17_b200 as mm
from torch.profiler import profile, ProfilerActivity
level = sys.argv[1] if len(sys.argv) > 1 else "unordered"
q = bench.ordered_workload(0, 1) if level == "ordered" else bench.unordered_workload(0)
n = len(q.recv_hdr)
sem = mm.MM_SEM_NOWILD_ORDERED if level == "ordered" else mm.MM_SEM_NOWILD_UNORDERED
eng = mm.Engine(sem, 1, n, n)
rh, mh = bench.to_dev(q.recv_hdr), bench.to_dev(q.msg_hdr)
orc = torch.empty(n, dtype=torch.int64, device="cuda"); omc = torch.empty_like(orc)
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
def step():
    eng.reset(); eng.post_recvs(rh); eng.push_msgs(mh); eng.match_batch(orc, omc, cnt)
for _ in range(3): step()
torch.cuda.synchronize()
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    step(); torch.cuda.synchronize()
evs = sorted([e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA], key=lambda e: e.time_range.start)
t0 = evs[0].time_range.start; prev = t0
for e in evs:
    s, d = e.time_range.start, e.time_range.end - e.time_range.start
    print("%8.1f  gap %7.1f  dur %7.1f  %s" % (s - t0, s - prev, d, e.name[:70]))
    prev = e.time_range.end
