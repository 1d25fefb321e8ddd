#!/usr/bin/env python
"""Per-kernel device time of one bench level via torch.profiler (CUPTI activity
records, no replay): a diagnostic split, not a bench number.
    python tools/kernel_split.py [mpi|ordered|unordered] [steps]
"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import bench
import paper_conf_ipps_klenkfed17_b200 as mm

level = sys.argv[1] if len(sys.argv) > 1 else "ordered"
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
torch.cuda.set_device(0)
if level == "mpi":
    q = bench.mpi_workload(0)
    eng = mm.Engine(mm.MM_SEM_MPI, q.n_endpoints, 1024, 1024)
    rh, mh, ro, mo = bench.to_dev(q.recv_hdr), bench.to_dev(q.msg_hdr), bench.to_dev(q.recv_off), bench.to_dev(q.msg_off)
    n = len(q.recv_hdr)
    def step():
        eng.reset(); eng.post_recvs(rh, None, ro); eng.push_msgs(mh, None, mo); eng.match_batch(orc, omc, cnt)
else:
    q = bench.ordered_workload(0, 1) if level == "ordered" else bench.unordered_workload(0)
    n = len(q.recv_hdr)
    sem = mm.MM_SEM_NOWILD_ORDERED if level == "ordered" else mm.MM_SEM_NOWILD_UNORDERED
    eng = mm.Engine(sem, 1, n, n, flat_kernel=int(os.environ.get("FLAT", "0")))
    rh, mh = bench.to_dev(q.recv_hdr), bench.to_dev(q.msg_hdr)
    def step():
        eng.reset(); eng.post_recvs(rh); eng.push_msgs(mh); eng.match_batch(orc, omc, cnt)
orc = torch.empty(n, dtype=torch.int64, device="cuda"); omc = torch.empty_like(orc)
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
for _ in range(3):
    step()
torch.cuda.synchronize()
from torch.profiler import profile, ProfilerActivity
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    for _ in range(steps):
        step()
    torch.cuda.synchronize()
tot = {}
for ev in prof.events():
    if ev.device_type == torch.autograd.DeviceType.CUDA:
        k = ev.name[:90]
        t = ev.device_time_total if hasattr(ev, "device_time_total") else ev.cuda_time_total
        c = tot.setdefault(k, [0, 0.0]); c[0] += 1; c[1] += t
all_t = sum(v[1] for v in tot.values())
print("%s: %.1f us per step on the device (%d steps)" % (level, all_t / steps, steps))
for k, (c, t) in sorted(tot.items(), key=lambda kv: -kv[1][1]):
    print("%8.1f us/step  %5.1f%%  x%-3d %s" % (t / steps, 100 * t / all_t, c // steps, k))
