# sweep kPartItems (partition items per lane) and time the no-wildcard levels; usage: bash tools/gpu_part_sweep.sh "8 4 6"
cd $GRAFT_REPO_ROOT
for it in ${1:-8 4 6}; do
  sed -i "s/^constexpr int kPartItems = [0-9]*;/constexpr int kPartItems = $it;/" paper_conf_ipps_klenkfed17_b200/csrc/mm_internal.cuh
  python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(force=True)" > /dev/null 2>&1 || { echo build failed; continue; }
  echo "== kPartItems $it"
  for l in ordered unordered; do timeout 300 python tools/kernel_split.py $l 5 2>&1 | grep -v -i warn | head -5; done
done
