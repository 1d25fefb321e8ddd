#!/usr/bin/env python
"""MPI-level host-buffer pipeline diagnostics: e2e ms/step per MM_OPT_PIPELINE_CHUNKS
value, raw H2D/D2H copy rates (alone and concurrent), and the copy/kernel
timeline of one pipelined step (torch.profiler)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from torch.profiler import ProfilerActivity, profile

import bench
import paper_conf_ipps_klenkfed17_b200 as mm
from paper_conf_ipps_klenkfed17_b200._lib import MM_OPT_PIPELINE_CHUNKS

q = bench.mpi_workload(0)
n_r = len(q.recv_hdr)
pin = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.int64).copy()).pin_memory()
rh, mh, ro, mo = pin(q.recv_hdr), pin(q.msg_hdr), pin(q.recv_off), pin(q.msg_off)
orc = torch.empty(n_r, dtype=torch.int64).pin_memory()
omc = torch.empty(n_r, dtype=torch.int64).pin_memory()
cnt = torch.zeros(2, dtype=torch.int64).pin_memory()
eng = mm.Engine(mm.MM_SEM_MPI, q.n_endpoints, 1024, 1024,
                host_out=mm.MM_HOST_OUT_MAPPED if os.environ.get("E2E_MAPPED") else None)


def step():
    eng.reset()
    eng.post_recvs(rh, None, ro)
    eng.push_msgs(mh, None, mo)
    eng.match_batch(orc, omc, cnt)


def t_ms(fn, k=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(k):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / k


for c in [1, 2, 4, 6, 8, 12, 16, 24, 32] if not os.environ.get("E2E_ONLY") else [4, 6, 8, 10, 12]:
    eng.set_option(MM_OPT_PIPELINE_CHUNKS, c)
    print("chunks %2d  e2e %.3f ms/step" % (c, t_ms(step)))
if os.environ.get("E2E_ONLY"):
    sys.exit(0)

# raw copy rates
dev = torch.empty(2 * n_r, dtype=torch.int64, device="cuda")
hin = torch.cat([rh, mh]).pin_memory()
hout = torch.empty(2 * n_r, dtype=torch.int64).pin_memory()
nb = 16 * n_r
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
h2d = t_ms(lambda: dev.copy_(hin, non_blocking=True))
d2h = t_ms(lambda: hout.copy_(dev, non_blocking=True))


def both():
    cur = torch.cuda.current_stream()
    s1.wait_stream(cur)
    s2.wait_stream(cur)
    with torch.cuda.stream(s1):
        dev[:n_r].copy_(hin[:n_r], non_blocking=True)
    with torch.cuda.stream(s2):
        hout[n_r:].copy_(dev[n_r:], non_blocking=True)
    cur.wait_stream(s1)
    cur.wait_stream(s2)


bo = t_ms(both)
print("H2D %.1f GB/s  D2H %.1f GB/s  (%d MB each)" % (nb / h2d / 1e6, nb / d2h / 1e6, nb >> 20))
print("concurrent H2D+D2H of %d MB each: %.3f ms (%.1f GB/s per direction)" % (nb >> 21, bo, nb / 2 / bo / 1e6))

eng.set_option(MM_OPT_PIPELINE_CHUNKS, int(os.environ.get("TL_CHUNKS", "6")))
step()
torch.cuda.synchronize()
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    step()
    step()
    torch.cuda.synchronize()
evs = sorted([e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA],
             key=lambda e: e.time_range.start)
t0 = evs[0].time_range.start
for e in evs:
    s, d = e.time_range.start, e.time_range.end - e.time_range.start
    print("%8.1f  dur %7.1f  %s" % (s - t0, d, e.name[:60]))
