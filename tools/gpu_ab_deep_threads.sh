# A/B of MM_DEEP_THREADS on configs[4] (mpi_worst level), alternating builds
cd $GRAFT_REPO_ROOT
for t in 512 1024; do MM_AB_DEFINES="MM_DEEP_THREADS=$t" python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(variant='deep$t')" > /dev/null 2>&1; done
for r in 1 2; do for t in 512 1024; do
MM_LIB=$GRAFT_REPO_ROOT/paper_conf_ipps_klenkfed17_b200/lib/libmm_deep$t.so timeout 300 python bench.py --levels mpi_worst --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); v=d['levels']['mpi_worst']; print('threads $t', round(v['value']/1e6,2), 'M/s', round(v['roofline']['kernel_ms'],4))"
done; done
