"""Per-phase cycle split of k_mpi_fifo on configs[1] (profiling aid).
Run on the GPU box after: python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(variant='timing')"
"""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["MM_LIB"] = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                    "paper_conf_ipps_klenkfed17_b200", "lib", "libmm_timing.so")
import numpy as np, torch
import synth
import paper_conf_ipps_klenkfed17_b200 as mm
from paper_conf_ipps_klenkfed17_b200 import _lib
L = _lib.load(build_if_missing=False)
L.mm_debug_phase_cycles.argtypes = [ctypes.c_void_p, ctypes.c_int]
q = synth.proxy_endpoints(seed=1)
if os.environ.get("N_EP"):
    q = q.subset(range(int(os.environ["N_EP"])))
dev = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.int64).copy()).cuda()
rh, mh, ro, mo = dev(q.recv_hdr), dev(q.msg_hdr), dev(q.recv_off), dev(q.msg_off)
n = len(q.recv_hdr)
orc = torch.empty(n, dtype=torch.int64, device="cuda"); omc = torch.empty_like(orc)
eng = mm.Engine(mm.MM_SEM_MPI, q.n_endpoints, 1024, 1024)
buf = np.zeros(16, np.uint64)
for it in range(3):
    eng.reset(); eng.post_recvs(rh, None, ro); eng.push_msgs(mh, None, mo); eng.match_batch(orc, omc)
    torch.cuda.synchronize()
    L.mm_debug_phase_cycles(buf.ctypes.data, 1)
tot = buf[:12].sum()
names = ["prologue", "P1 stage", "P2 insert", "P3 ids", "P4 classify", "P5 scans", "P6 place", "P7 wildcards",
         "P8 resolve+out", "P9 msg compact", "P7a group setup", "P7 K<=32 chain"]
for i, nm in enumerate(names):
    print("%-16s %8.0f cycles/endpoint  %5.1f%%" % (nm, buf[i] / q.n_endpoints, 100.0 * buf[i] / tot))
print("total %.0f cycles per endpoint (per CTA, thread 0)" % (tot / q.n_endpoints))
print("endpoints on the K<=32 chain: %d, on the group path: %d" % (buf[13], buf[14]))

# per-endpoint P7 (wildcard phase) cycles by class
L.mm_debug_ep.argtypes = [ctypes.c_void_p, ctypes.c_int]
dbg = np.zeros(4 * q.n_endpoints, np.uint32)
L.mm_debug_ep(dbg.ctypes.data, q.n_endpoints)
dbg = dbg.reshape(-1, 4).astype(np.int64)
cyc, K, W, G = dbg.T
for lo, hi, nm in [(0, 33, "K<=32"), (33, 200, "K 33-199"), (200, 600, "K 200-599"), (600, 2000, "K>=600")]:
    m = (K >= lo) & (K < hi)
    if m.any():
        print("%-10s n=%4d  P7 %7.0f cyc  K %6.1f  W %5.1f  groups %5.1f  cyc/wildcard %5.0f" % (
            nm, m.sum(), cyc[m].mean(), K[m].mean(), W[m].mean(), G[m].mean(), (cyc[m] / np.maximum(W[m], 1)).mean()))
