"""Per-phase cycle split of k_bucket_match (no-wildcard levels) -- a
profiling aid.  Run on the GPU box after:
python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(variant='timing')"
usage: python tools/bucket_phase_timing.py [ordered|unordered]
"""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["MM_LIB"] = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                    "paper_conf_ipps_klenkfed17_b200", "lib", "libmm_timing.so")
import numpy as np, torch
import bench
import paper_conf_ipps_klenkfed17_b200 as mm
from paper_conf_ipps_klenkfed17_b200 import _lib
level = sys.argv[1] if len(sys.argv) > 1 else "ordered"
L = _lib.load(build_if_missing=False)
L.mm_debug_bucket_cycles.argtypes = [ctypes.c_void_p, ctypes.c_int]
q = bench.ordered_workload(0, 1) if level == "ordered" else bench.unordered_workload(0)
n = len(q.recv_hdr)
sem = mm.MM_SEM_NOWILD_ORDERED if level == "ordered" else mm.MM_SEM_NOWILD_UNORDERED
eng = mm.Engine(sem, 1, n, n)
rh, mh = bench.to_dev(q.recv_hdr), bench.to_dev(q.msg_hdr)
orc = torch.empty(n, dtype=torch.int64, device="cuda"); omc = torch.empty_like(orc)
buf = np.zeros(16, np.uint64)
for it in range(3):
    eng.reset(); eng.post_recvs(rh); eng.push_msgs(mh); eng.match_batch(orc, omc)
    torch.cuda.synchronize()
    L.mm_debug_bucket_cycles(buf.ctypes.data, 1)
nb = max(1, int(buf[15]))
tot = buf[:8].sum()
names = ["top barrier (wait)", "A load+clear", "B table insert", "C ids+counts", "D group scan", "E place",
         "F order by index", "G pair+out"]
for i, nm in enumerate(names):
    print("%-20s %8.0f cycles/bucket  %5.1f%%" % (nm, buf[i] / nb, 100.0 * buf[i] / tot))
print("total %.0f cycles per bucket (thread 0), %d buckets" % (tot / nb, nb))
