# MPI-level tests (incl. the randomised sweep), phase timing and two bench lines
cd $GRAFT_REPO_ROOT
python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(force=True); _build.build_library(variant='timing')" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -k "mpi or smoke" 2>&1 | tail -1
python tools/phase_timing.py 2>&1 | tail -6
for i in 1 2; do timeout 300 python bench.py --levels mpi --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('mpi', round(d['value']/1e9,3), d['roofline']['kernel_ms'])"; done
