cd $GRAFT_REPO_ROOT
F=paper_conf_ipps_klenkfed17_b200/csrc/k_mpi_fifo.cu
for t in 512 1024; do
  sed -i "s/^#define MM_DEEP_THREADS [0-9]*/#define MM_DEEP_THREADS $t/" $F
  python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(force=True)" > /dev/null 2>&1
  grep -A2 "k_mpi_fifoILi${t}ELb0" paper_conf_ipps_klenkfed17_b200/lib/ptxas.log | grep spill | head -1
  echo "threads $t: $(python tools/config4_time.py 2>&1 | tail -1)"
done
