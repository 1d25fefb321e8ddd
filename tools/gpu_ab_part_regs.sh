# A/B of the scatter kernel's register budget (resident CTAs per SM)
cd $GRAFT_REPO_ROOT
for m in 3 4; do
  sed -i "s/^#define MM_PART_MIN_BLOCKS [0-9]*/#define MM_PART_MIN_BLOCKS $m/" paper_conf_ipps_klenkfed17_b200/csrc/mm_internal.cuh
  python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(force=True)" > /dev/null 2>&1
  grep -A2 "k_part_scatter" paper_conf_ipps_klenkfed17_b200/lib/ptxas.log | grep -i "registers\|spill" | head -2
  for i in 1 2; do timeout 600 python bench.py --levels ordered,unordered --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('min $m', ' '.join('%s %.3f %.4f' % (k, v['value']/1e9, v['roofline']['kernel_ms']) for k, v in d['levels'].items()))"; done
done
