# A/B of the scatter's items per lane x resident CTAs per SM
cd $GRAFT_REPO_ROOT
F=paper_conf_ipps_klenkfed17_b200/csrc/mm_internal.cuh
for cfg in "6 4" "4 5" "5 5" "4 6"; do
  set -- $cfg
  sed -i "s/^constexpr int kPartItems = [0-9]*;/constexpr int kPartItems = $1;/" $F
  sed -i "s/^#define MM_PART_MIN_BLOCKS [0-9]*/#define MM_PART_MIN_BLOCKS $2/" $F
  python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(force=True)" > /dev/null 2>&1 || { echo "build fail $cfg"; continue; }
  grep -A2 "k_part_scatter" paper_conf_ipps_klenkfed17_b200/lib/ptxas.log | grep -i "spill" | head -1
  for i in 1 2; do timeout 600 python bench.py --levels ordered,unordered --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('items/min $cfg', ' '.join('%s %.3f %.4f' % (k, v['value']/1e9, v['roofline']['kernel_ms']) for k, v in d['levels'].items()))"; done
done
