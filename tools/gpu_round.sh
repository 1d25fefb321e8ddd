# Full round evidence: gpu tests, smoke, bench (with cpu baselines), per-level ncu traffic,
# ncu launch list, ncu --set full of the top kernels (summarised on the box; the large
# .ncu-rep files are deleted so that gpurun_out stays under its 64 MiB cap).
# usage: bash tools/gpu_round.sh <tag> [skip_tests]
cd $GRAFT_REPO_ROOT
TAG=${1:-x}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1 || { tail -20 gpurun_out/build_$TAG.log; exit 1; }
cp paper_conf_ipps_klenkfed17_b200/lib/ptxas.log gpurun_out/ptxas_$TAG.log
if [ -z "$2" ]; then
timeout 1500 python -m pytest tests -m gpu -q --maxfail=5 -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1; tail -2 gpurun_out/pytest_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
fi
timeout 900 python bench.py > gpurun_out/bench_$TAG.log 2>&1; tail -1 gpurun_out/bench_$TAG.log | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('clocks', d['clocks'])
for k,v in d['levels'].items(): print(k, round(v['value']/1e9,3), 'Gm/s', round(v['ms_per_step'],3), 'ms kernel', round(v['roofline']['kernel_ms'],3), 'frac', round(v['roofline']['frac'],4))"
bash tools/gpu_level_traffic.sh $TAG > gpurun_out/level_traffic_$TAG.txt 2>&1; cat gpurun_out/level_traffic_$TAG.txt
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --levels mpi,mpi_cookies,mpi_matrix,ordered,unordered,mpi_worst > gpurun_out/ncu_launch_$TAG.log 2>&1
python tools/ncu_summary.py launches gpurun_out/launches_$TAG.csv gpurun_out/launches_$TAG.md > /dev/null
# device-input launches only (the e2e leg's pipelined launches cover a part of the endpoints each)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_mpi_fifo" -s 3 -c 1 -o gpurun_out/prof_mpi_$TAG \
    python bench.py --steps 1 --warmup 3 --levels mpi --no-cpu-baseline > gpurun_out/ncu_mpi_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_mpi_matrix" -s 3 -c 1 -o gpurun_out/prof_mpim_$TAG \
    python bench.py --steps 1 --warmup 3 --levels mpi_matrix --no-cpu-baseline > gpurun_out/ncu_mpim_$TAG.log 2>&1
# one whole step of each relaxed level (every launch of the engine's timed region)
timeout 900 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include "mm_timed:ordered/mm_region]" -o gpurun_out/prof_flat_$TAG \
    python bench.py --steps 1 --warmup 3 --levels ordered --no-cpu-baseline --nvtx > gpurun_out/ncu_flat_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include "mm_timed:unordered/mm_region]" -o gpurun_out/prof_pop_$TAG \
    python bench.py --steps 1 --warmup 3 --levels unordered --no-cpu-baseline --nvtx > gpurun_out/ncu_pop_$TAG.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_mpi_fifo" -s 3 -c 1 -o gpurun_out/prof_deep_$TAG \
    python bench.py --steps 1 --warmup 3 --levels mpi_worst --no-cpu-baseline > gpurun_out/ncu_deep_$TAG.log 2>&1
T=gpurun_out/kernel_traffic_$TAG.json
python tools/ncu_summary.py full gpurun_out/prof_mpi_$TAG.ncu-rep gpurun_out/ncu_mpi_$TAG.md --traffic $T > /dev/null
python tools/ncu_summary.py full gpurun_out/prof_mpim_$TAG.ncu-rep gpurun_out/ncu_mpi_matrix_$TAG.md --traffic $T > /dev/null
python tools/ncu_summary.py full gpurun_out/prof_flat_$TAG.ncu-rep gpurun_out/ncu_ordered_$TAG.md > /dev/null
python tools/ncu_summary.py full gpurun_out/prof_pop_$TAG.ncu-rep gpurun_out/ncu_unordered_$TAG.md > /dev/null
python tools/ncu_summary.py full gpurun_out/prof_deep_$TAG.ncu-rep gpurun_out/ncu_mpi_deep_$TAG.md --traffic $T --key k_mpi_fifo_deep > /dev/null
rm -f gpurun_out/prof_flat_$TAG.ncu-rep gpurun_out/prof_pop_$TAG.ncu-rep gpurun_out/prof_mpim_$TAG.ncu-rep
du -sh gpurun_out; ls gpurun_out | grep $TAG
