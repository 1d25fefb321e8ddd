#!/usr/bin/env python
"""Kernel/copy timeline of two steps of a no-wildcard bench level (torch
profiler, CUPTI): where the GPU time of a step goes outside the timed region.
    python tools/step_timeline.py [ordered|unordered]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from torch.profiler import ProfilerActivity, profile

import bench
import paper_conf_ipps_klenkfed17_b200 as mm

level = sys.argv[1] if len(sys.argv) > 1 else "ordered"
q = bench.ordered_workload(0, 1) if level == "ordered" else bench.unordered_workload(0)
n = len(q.recv_hdr)
rh, mh = bench.to_dev(q.recv_hdr), bench.to_dev(q.msg_hdr)
sem = mm.MM_SEM_NOWILD_ORDERED if level == "ordered" else mm.MM_SEM_NOWILD_UNORDERED
eng = mm.Engine(sem, 1, n, n)
orc = torch.empty(n, dtype=torch.int64, device="cuda")
omc = torch.empty_like(orc)
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")


def step():
    eng.reset()
    eng.post_recvs(rh)
    eng.push_msgs(mh)
    eng.match_batch(orc, omc, cnt)


for _ in range(5):
    step()
torch.cuda.synchronize()
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    for _ in range(3):
        step()
    torch.cuda.synchronize()
evs = sorted([e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA],
             key=lambda e: e.time_range.start)
t0 = evs[0].time_range.start
prev_end = t0
for e in evs:
    s, d = e.time_range.start, e.time_range.end - e.time_range.start
    print("%8.1f  gap %6.1f  dur %7.1f  %s" % (s - t0, s - prev_end, d, e.name[:70]))
    prev_end = max(prev_end, e.time_range.end)

# host time per API call of a step (a call that waits for the GPU shows ~a step)
import time
torch.cuda.synchronize()
acc = {"reset": 0.0, "post": 0.0, "push": 0.0, "match": 0.0}
K = 20
for _ in range(K):
    t = time.perf_counter(); eng.reset(); acc["reset"] += time.perf_counter() - t
    t = time.perf_counter(); eng.post_recvs(rh); acc["post"] += time.perf_counter() - t
    t = time.perf_counter(); eng.push_msgs(mh); acc["push"] += time.perf_counter() - t
    t = time.perf_counter(); eng.match_batch(orc, omc, cnt); acc["match"] += time.perf_counter() - t
torch.cuda.synchronize()
print("host us per call:", {k: round(v / K * 1e6, 1) for k, v in acc.items()})
