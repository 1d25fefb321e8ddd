# configs[4] per-phase cycles (timing build)
cd $GRAFT_REPO_ROOT
python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(force=True); _build.build_library(variant='timing')" > /dev/null 2>&1
timeout 300 python tools/config4_phase.py 2>&1 | tail -14
