# 2 ranks sharing one GPU over gloo: exercises bench.py's N>1 path (timing not meaningful)
cd $GRAFT_REPO_ROOT
MM_BENCH_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29555 \
   bench.py --gpus 2 --steps 2 --warmup 3 --levels mpi,ordered,unordered > gpurun_out/bench_mr.log 2>&1
echo rc=$?; tail -3 gpurun_out/bench_mr.log | cut -c1-600
