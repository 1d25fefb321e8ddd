# A/B of MM_STAGE_WLOG on configs[4] (mpi_worst level), alternating builds
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "mpi or smoke or fuzz" 2>&1 | tail -1
for c in 0 1; do MM_AB_DEFINES="MM_STAGE_WLOG=$c" python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(variant='wlog$c')" > /dev/null 2>&1; done
for r in 1 2 3; do for c in 0 1; do
MM_LIB=$GRAFT_REPO_ROOT/paper_conf_ipps_klenkfed17_b200/lib/libmm_wlog$c.so timeout 300 python bench.py --levels mpi_worst --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); v=d['levels']['mpi_worst']; print('wlog $c', round(v['value']/1e6,2), 'M/s', round(v['roofline']['kernel_ms'],4))"
done; done
