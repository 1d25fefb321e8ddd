# A/B of k_bucket_pop's minimum resident CTAs (register budget)
cd $GRAFT_REPO_ROOT
for m in 5 6 7; do
  sed -i "s/^#define MM_POP_MIN_BLOCKS [0-9]*/#define MM_POP_MIN_BLOCKS $m/" paper_conf_ipps_klenkfed17_b200/csrc/k_bucket.cu
  python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(force=True)" > /dev/null 2>&1
  grep -A3 "k_bucket_pop" paper_conf_ipps_klenkfed17_b200/lib/ptxas.log | grep -i "registers" | head -1
  for i in 1 2; do timeout 600 python bench.py --levels unordered --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); v=d['levels']['unordered']; print('min blocks $m', round(v['value']/1e9,3), round(v['roofline']['kernel_ms'],3))"; done
done
