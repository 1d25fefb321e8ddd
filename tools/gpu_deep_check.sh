# deep-endpoint (global workspace) parity subset + configs[4] bench
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "lead or worst or maximum or deep or config4 or fuzz or wide or contract" 2>&1 | tail -4
timeout 300 python bench.py --levels mpi_worst,mpi --no-cpu-baseline > gpurun_out/b.log 2>&1; tail -1 gpurun_out/b.log | python -c "
import json,sys; d=json.loads(sys.stdin.read())
for k,v in d['levels'].items(): print(k, round(v['value']/1e9,4), 'Gm/s', round(v['ms_per_step'],4), 'ms kernel', round(v['roofline']['kernel_ms'],4), v.get('step_value'))"
