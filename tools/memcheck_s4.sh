# compute-sanitizer memcheck of the kernels added late in round 1:
# pc_waitall_on_stream's wait_all_kernel and the two-level aggregation counters.
# usage: gpurun --timeout 1500 -- "bash tools/memcheck_s4.sh"
mkdir -p gpurun_out
PC_TIMEOUT_MS=60000 timeout 1200 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest -q -x \
  tests/test_gpu_waitall.py \
  "tests/test_gpu_p2p.py::test_two_level_aggregation_counters" > gpurun_out/memcheck_s4.txt 2>&1
tail -4 gpurun_out/memcheck_s4.txt
