# no-wildcard levels: parity subset + bench + per-kernel ncu of one step
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "ordered or unordered or nowild or flat or bucket or world2 or smoke" 2>&1 | tail -4
timeout 300 python bench.py --levels ordered,unordered,unordered_256m --no-cpu-baseline > gpurun_out/b.log 2>&1; tail -1 gpurun_out/b.log | python -c "
import json,sys; d=json.loads(sys.stdin.read())
for k,v in d['levels'].items(): print(k, round(v['value']/1e9,3), 'Gm/s', round(v['ms_per_step'],3), 'ms kernel', round(v['roofline']['kernel_ms'],3), v.get('bucket_fallbacks'))"
for L in ordered unordered; do timeout 600 ncu --nvtx --nvtx-include "mm_timed:$L/mm_region]" --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/q_$L.csv python bench.py --levels $L --steps 1 --warmup 3 --no-cpu-baseline --nvtx > /dev/null 2>&1; done
python tools/level_traffic.py gpurun_out/lt.json ordered=gpurun_out/q_ordered.csv unordered=gpurun_out/q_unordered.csv > /dev/null
python -c "
import json
d=json.load(open('gpurun_out/lt.json'))
for L,v in d.items():
    print(L, '%.0f MB' % (v['region_dram_bytes_per_step']/1e6))
    for k,x in v['region_kernels'].items(): print('   ', k, x['launches'], '%.1f MB' % (x['dram_bytes']/1e6), '%.1f us' % x['us'])"
