"""Per-phase cycles of k_mpi_fifo on configs[4] (one 16K-deep endpoint) from
the timing build (profiling aid)."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["MM_LIB"] = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                    "paper_conf_ipps_klenkfed17_b200", "lib", "libmm_timing.so")
import numpy as np, torch
import synth, bench
import paper_conf_ipps_klenkfed17_b200 as mm
from paper_conf_ipps_klenkfed17_b200 import _lib
L = _lib.load(build_if_missing=False)
L.mm_debug_phase_cycles.argtypes = [ctypes.c_void_p, ctypes.c_int]
q = synth.worst_chain()
n = len(q.recv_hdr)
eng = mm.Engine(mm.MM_SEM_MPI, 1, n, n)
rh, mh, ro, mo = bench.to_dev(q.recv_hdr), bench.to_dev(q.msg_hdr), bench.to_dev(q.recv_off), bench.to_dev(q.msg_off)
orc = torch.empty(n, dtype=torch.int64, device="cuda"); omc = torch.empty_like(orc)
buf = np.zeros(16, np.uint64)
for it in range(3):
    eng.reset(); eng.post_recvs(rh, None, ro); eng.push_msgs(mh, None, mo); eng.match_batch(orc, omc)
    torch.cuda.synchronize()
    L.mm_debug_phase_cycles(buf.ctypes.data, 1)
names = ["prologue", "P1 stage", "P2 insert", "P7 lead: messages", "P4 classify", "P5 scans", "P6 place",
         "P7 wildcards", "P8 resolve+out", "P9 msg compact", "P7a group setup", "P7 K<=32 chain", "P7 lead: fe",
         "-", "-", "P7 lead: run ranks"]
tot = buf[:13].sum() + buf[15]
for i, nm in enumerate(names):
    if nm != "-":
        print("%-20s %9.0f cycles  %5.1f%%" % (nm, buf[i], 100.0 * buf[i] / max(tot, 1)))
print("total %.0f cycles (one endpoint), K<=32 chain %d, group path %d" % (tot, buf[13], buf[14]))
