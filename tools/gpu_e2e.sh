#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 600 python bench.py --steps 20 --warmup 5 --no-latency --no-jacobi --no-c1 --no-cpu-baseline > gpurun_out/r02_bench_e2e.json 2> gpurun_out/r02_bench_e2e.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29655 \
  bench.py --gpus 2 --steps 5 --warmup 3 --no-c1 --no-jacobi --no-dl > gpurun_out/multi_bench.log 2> gpurun_out/multi_bench.err; echo "bench exit $?" >> gpurun_out/multi_bench.err
tail -3 gpurun_out/r02_bench_e2e.err; tail -2 gpurun_out/multi_bench.err
