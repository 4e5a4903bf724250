# The N > 1 path on a one-GPU box: cross-process parity test, then bench.py
# under torchrun with 2 ranks sharing cuda:0 (gloo bootstrap, no NCCL baseline).
# usage: gpurun --timeout 900 -- "bash tools/gpu_multi_check.sh"
mkdir -p gpurun_out
timeout 400 python -m pytest tests/test_gpu_multiproc.py -x -q > gpurun_out/multi_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/multi_pytest.log
timeout 400 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29655 \
  bench.py --gpus 2 --steps 20 --warmup 3 --bytes 16777216 --quiet > gpurun_out/multi_bench.log 2>&1; echo "bench exit $?" >> gpurun_out/multi_bench.log
tail -3 gpurun_out/multi_pytest.log; tail -c 1500 gpurun_out/multi_bench.log
