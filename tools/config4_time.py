"""configs[4] (worst-case chain: one endpoint, 16K-deep queues, leading
ANY_SOURCE receives): device time of one batch vs the C oracle (diagnostic)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth, oracle, bench
import paper_conf_ipps_klenkfed17_b200 as mm
q = synth.worst_chain()
n = len(q.recv_hdr)
eng = mm.Engine(mm.MM_SEM_MPI, 1, n, n)
rh, mh, ro, mo = bench.to_dev(q.recv_hdr), bench.to_dev(q.msg_hdr), bench.to_dev(q.recv_off), bench.to_dev(q.msg_off)
orc = torch.empty(n, dtype=torch.int64, device="cuda"); omc = torch.empty_like(orc)
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
def step():
    eng.reset(); eng.post_recvs(rh, None, ro); eng.push_msgs(mh, None, mo); eng.match_batch(orc, omc, cnt)
for _ in range(3): step()
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(10): step()
b.record(); torch.cuda.synchronize()
ms = a.elapsed_time(b) / 10
m = int(cnt[1])
oracle.lib()
t0 = time.perf_counter(); mr, _ = oracle.mpi_endpoints(q); t = time.perf_counter() - t0
print("configs[4]: %d matches; GPU %.3f ms per batch (%.1f M matches/s); oracle %.3f ms (%.1f M matches/s)" % (
    m, ms, m / ms / 1e3, t * 1e3, int((mr >= 0).sum()) / t / 1e6))
