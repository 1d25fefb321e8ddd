cd $GRAFT_REPO_ROOT
TAG=${1:-x}
timeout 1200 python -m pytest tests -m gpu -q --maxfail=5 -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1; tail -2 gpurun_out/pytest_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 600 python bench.py --levels mpi,ordered,unordered --no-cpu-baseline > gpurun_out/bench_$TAG.log 2>&1; tail -1 gpurun_out/bench_$TAG.log | python -c "
import json,sys; d=json.loads(sys.stdin.read())
for k,v in d['levels'].items(): print(k, round(v['value']/1e9,3), 'Gm/s', round(v['ms_per_step'],3), 'ms kernel', round(v['roofline']['kernel_ms'],3), 'frac', round(v['roofline']['frac'],4))"
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
    python bench.py --steps 1 --warmup 3 --levels mpi,ordered,unordered --no-cpu-baseline > /dev/null 2>&1
