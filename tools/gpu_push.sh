#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_direct_push.py tests/test_gpu_batch.py tests/test_gpu_overlap.py tests/test_gpu_allreduce.py -x -q 2>&1 | tail -15 > gpurun_out/r02_push_pytest.txt
timeout 600 python bench.py --steps 20 --warmup 5 --algo direct_push --no-latency --no-jacobi --no-c1 --no-cpu-baseline > gpurun_out/r02_bench_push.json 2> gpurun_out/r02_bench_push.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29655 \
  bench.py --gpus 2 --steps 5 --warmup 3 --no-c1 --no-jacobi > gpurun_out/multi_bench.log 2> gpurun_out/multi_bench.err; echo "bench exit $?" >> gpurun_out/multi_bench.err
tail -3 gpurun_out/r02_push_pytest.txt; cut -c1-300 gpurun_out/r02_bench_push.json; tail -2 gpurun_out/multi_bench.err
