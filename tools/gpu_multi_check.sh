# The N > 1 path on a one-GPU box: cross-process parity test, then bench.py
# with 2 ranks sharing cuda:0 (gloo bootstrap, no NCCL baseline): once
# self-launched (`python bench.py --gpus 2` re-execs under torchrun) and once
# under torchrun directly (the driver's launch).
# usage: gpurun --timeout 900 -- "bash tools/gpu_multi_check.sh"
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 400 python -m pytest tests/test_gpu_multiproc.py -x -q > gpurun_out/multi_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/multi_pytest.log
timeout 900 python bench.py --gpus 2 --steps 5 --warmup 3 > gpurun_out/multi_bench_self.log 2> gpurun_out/multi_bench_self.err; echo "bench exit $?" >> gpurun_out/multi_bench_self.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29655 \
  bench.py --gpus 2 --steps 5 --warmup 3 > gpurun_out/multi_bench.log 2> gpurun_out/multi_bench.err; echo "bench exit $?" >> gpurun_out/multi_bench.err
tail -3 gpurun_out/multi_pytest.log; tail -c 1500 gpurun_out/multi_bench_self.log; tail -2 gpurun_out/multi_bench_self.err; tail -c 600 gpurun_out/multi_bench.log; tail -2 gpurun_out/multi_bench.err
