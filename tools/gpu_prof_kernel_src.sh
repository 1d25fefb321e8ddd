# ncu --set full + per-source-line profile of one kernel (regex) of a bench level
# usage: bash tools/gpu_prof_kernel_src.sh <tag> <kernel-regex> <level> [skip]
cd $GRAFT_REPO_ROOT
TAG=${1:-x}; KR=${2:-k_part_scatter}; LV=${3:-ordered}; SK=${4:-3}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1 || { tail -20 gpurun_out/build_$TAG.log; exit 1; }
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"$KR" -s $SK -c 1 -o gpurun_out/prof_$TAG \
    python bench.py --steps 1 --warmup 3 --levels $LV --no-cpu-baseline > gpurun_out/ncu_$TAG.log 2>&1
ncu -i gpurun_out/prof_$TAG.ncu-rep --page source --csv --print-source cuda,sass -c 1 > gpurun_out/src_$TAG.csv 2>&1
python tools/ncu_lines.py gpurun_out/src_$TAG.csv 25
python tools/ncu_summary.py full gpurun_out/prof_$TAG.ncu-rep gpurun_out/sum_$TAG.md > /dev/null 2>&1; head -40 gpurun_out/sum_$TAG.md
