#!/bin/bash
# compute-sanitizer memcheck over the round-2 paths: overlap (early fork, thin
# engine), INLINE allreduce, batched epoch + engine, DIRECT PUSH, p2p engine
# sweep-fence; racecheck over the shared-memory epoch batch kernel.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
PC_TIMEOUT_MS=120000 timeout 1500 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest -q -x \
 "tests/test_gpu_overlap.py::test_engine_runs_while_producer_runs[3-4]" \
 "tests/test_gpu_overlap.py::test_engine_runs_while_producer_runs[1-3]" \
 "tests/test_gpu_inline_allreduce.py::test_inline_fp32_producer[0-4-1001-3]" \
 "tests/test_gpu_inline_allreduce.py::test_inline_fp32_producer[1-3-17-5]" \
 "tests/test_gpu_inline_allreduce.py::test_inline_host_pready_range" \
 "tests/test_gpu_batch.py::test_batched_per_tensor_fp32[epoch_all-4]" \
 "tests/test_gpu_batch.py::test_batched_falls_back_for_ring" \
 "tests/test_gpu_direct_push.py::test_push_fp32_bitexact[2-4099-3]" \
 "tests/test_gpu_direct_push.py::test_push_inplace_producer" \
 "tests/test_gpu_p2p.py::test_granularity_aggregation_copy[1-odd-0]" \
 "tests/test_gpu_p2p.py::test_granularity_aggregation_copy[1-none-2]" > gpurun_out/r02_memcheck.txt 2>&1
tail -4 gpurun_out/r02_memcheck.txt
PC_TIMEOUT_MS=120000 timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python -m pytest -q -x \
 "tests/test_gpu_batch.py::test_batched_per_tensor_fp32[epoch_all-2]" > gpurun_out/r02_racecheck.txt 2>&1
tail -4 gpurun_out/r02_racecheck.txt
