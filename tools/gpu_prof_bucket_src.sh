# ncu --set full + per-source-line profile of k_bucket_pair; usage: bash tools/gpu_prof_bucket_src.sh <tag> [ordered|unordered]
cd $GRAFT_REPO_ROOT
TAG=${1:-x}; LV=${2:-ordered}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1 || { tail -20 gpurun_out/build_$TAG.log; exit 1; }
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_bucket_pair" -s 3 -c 1 -o gpurun_out/prof_bp_$TAG \
    python bench.py --steps 1 --warmup 3 --levels $LV --no-cpu-baseline > gpurun_out/ncu_bp_$TAG.log 2>&1
ncu -i gpurun_out/prof_bp_$TAG.ncu-rep --page source --csv --print-source cuda,sass -k regex:k_bucket_pair -c 1 > gpurun_out/bp_src_$TAG.csv 2>&1
python tools/ncu_lines.py gpurun_out/bp_src_$TAG.csv 30
python tools/ncu_summary.py full gpurun_out/prof_bp_$TAG.ncu-rep gpurun_out/bp_sum_$TAG.md > /dev/null 2>&1; cat gpurun_out/bp_sum_$TAG.md | head -40
