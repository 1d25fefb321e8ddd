# ncu --set full of both partition passes of one ordered step + per-line stall table
cd $GRAFT_REPO_ROOT
TAG=${1:-x}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_part_pass" -s 6 -c 2 -o gpurun_out/prof_pass_$TAG \
    python bench.py --steps 1 --warmup 3 --levels ordered --no-cpu-baseline > gpurun_out/ncu_pass_$TAG.log 2>&1
ncu -i gpurun_out/prof_pass_$TAG.ncu-rep --page source --csv --print-source cuda,sass -k regex:k_part_pass -c 1 -s 1 > gpurun_out/src_pass_$TAG.csv 2>&1
python tools/ncu_stalls.py gpurun_out/src_pass_$TAG.csv 25
python tools/ncu_summary.py full gpurun_out/prof_pass_$TAG.ncu-rep gpurun_out/sum_pass_$TAG.md > /dev/null 2>&1; cat gpurun_out/sum_pass_$TAG.md | head -60
rm -f gpurun_out/prof_pass_$TAG.ncu-rep
