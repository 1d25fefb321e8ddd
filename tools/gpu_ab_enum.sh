# A/B of MM_ENUM_ONCHIP on the configs[1] MPI level, alternating builds
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for c in 0 1; do MM_AB_DEFINES="MM_ENUM_ONCHIP=$c" python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(variant='enum$c')" > /dev/null 2>&1; done
MM_LIB=$GRAFT_REPO_ROOT/paper_conf_ipps_klenkfed17_b200/lib/libmm_enum0.so timeout 600 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "mpi" 2>&1 | tail -1
for r in 1 2 3; do for c in 0 1; do
MM_LIB=$GRAFT_REPO_ROOT/paper_conf_ipps_klenkfed17_b200/lib/libmm_enum$c.so timeout 300 python bench.py --levels mpi --no-cpu-baseline --steps 50 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); v=d['levels']['mpi']; print('enum $c', round(v['value']/1e9,3), 'G/s', round(v['roofline']['kernel_ms'],4))"
done; done
