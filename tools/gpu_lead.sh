# leading-run check: MPI-level GPU tests + mpi / mpi_worst bench lines
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo build failed; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "mpi or smoke or fuzz" > gpurun_out/pytest_lead.log 2>&1; tail -3 gpurun_out/pytest_lead.log
for i in 1 2; do timeout 300 python bench.py --levels mpi,mpi_worst --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
for k,v in d['levels'].items(): print(k, round(v['value']/1e6,2), 'M/s kernel ms', round(v['roofline']['kernel_ms'],4), 'issue', v.get('issue',{}).get('frac'))"; done
python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(variant='timing')" > /dev/null 2>&1
timeout 300 python tools/config4_phase.py 2>&1 | tail -14
