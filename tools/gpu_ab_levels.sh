# A/B of any bench levels via MM_AB_DEFINES builds, twice each
# usage: LEVELS=ordered,unordered bash tools/gpu_ab_levels.sh "<defines A>" "<defines B>" ...
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do
for cfg in "$@"; do
  export MM_AB_DEFINES="$cfg"
  python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(variant='ab')" > /dev/null 2>&1 || { echo "build fail $cfg"; continue; }
  MM_LIB=$PWD/paper_conf_ipps_klenkfed17_b200/lib/libmm_ab.so timeout 900 python bench.py --levels ${LEVELS:-mpi} --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('$cfg', ' '.join('%s %.3f G/s %.4f ms/step %.4f kernel' % (k, v['value']/1e9, v['ms_per_step'], v['roofline']['kernel_ms']) for k, v in d['levels'].items()))"
done
done
