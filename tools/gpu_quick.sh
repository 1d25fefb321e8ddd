# quick iteration: build, GPU tests (optionally filtered), bench of chosen levels, phase timing
# usage: bash tools/gpu_quick.sh <tag> [pytest -k expr] [levels]
cd $GRAFT_REPO_ROOT
TAG=${1:-x}; K=${2:-}; LV=${3:-mpi}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1 || { tail -20 gpurun_out/build_$TAG.log; exit 1; }
if [ -n "$K" ]; then timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "$K" > gpurun_out/pytest_$TAG.log 2>&1;
else timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1; fi
tail -3 gpurun_out/pytest_$TAG.log; grep -m5 -B5 "Error\|assert" gpurun_out/pytest_$TAG.log | head -60
timeout 600 python bench.py --levels $LV --no-cpu-baseline > gpurun_out/bench_$TAG.log 2>&1; tail -1 gpurun_out/bench_$TAG.log | python -c "
import json,sys; d=json.loads(sys.stdin.read())
for k,v in d['levels'].items(): print(k, round(v['value']/1e9,3), 'Gm/s', round(v['ms_per_step'],3), 'ms kernel', round(v['roofline']['kernel_ms'],3), 'frac', round(v['roofline']['frac'],4), 'e2e', round(v['e2e']['value']/1e9,3) if 'e2e' in v else '', v.get('e2e',{}).get('ms_per_step',''))" || tail -5 gpurun_out/bench_$TAG.log
if [ -n "$PHASE" ]; then python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(variant='timing')" && python tools/phase_timing.py 2>&1 | tail -16; fi
