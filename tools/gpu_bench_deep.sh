# bench line + the configs[4] deep-launch ncu capture; logs under gpurun_out/
# usage: bash tools/gpu_bench_deep.sh <tag>
cd $GRAFT_REPO_ROOT
TAG=${1:-x}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1 || { tail -20 gpurun_out/build_$TAG.log; exit 1; }
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_mpi_fifo" -s 2 -c 1 -o gpurun_out/prof_deep_$TAG \
    python bench.py --steps 1 --warmup 3 --levels mpi_worst --no-cpu-baseline > gpurun_out/ncu_deep_$TAG.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_$TAG.log 2>&1; tail -1 gpurun_out/bench_$TAG.log | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('clocks', d['clocks'])
for k,v in d['levels'].items(): print(k, round(v['value']/1e9,4), 'Gm/s', round(v['ms_per_step'],3), 'ms kernel', round(v['roofline']['kernel_ms'],4))"
