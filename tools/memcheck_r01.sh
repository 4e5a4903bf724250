PC_TIMEOUT_MS=60000 timeout 1200 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest -q -x \
 "tests/test_gpu_jacobi.py::test_jacobi_bitexact_vs_oracle[rows-2-2-256]" \
 "tests/test_gpu_jacobi.py::test_jacobi_traditional_baseline_bitexact[2-2-512]" \
 "tests/test_gpu_p2p.py::test_xpart_different_partition_counts[1-2-6-4]" \
 "tests/test_gpu_p2p.py::test_xpart_different_partition_counts[0-1-8-3]" \
 "tests/test_gpu_p2p.py::test_host_progression_engine_tagged_epochs[4]" \
 "tests/test_gpu_allreduce.py::test_epoch_all_single_control_kernel[True-3-8]" \
 "tests/test_gpu_allreduce.py::test_direct_ragged_inplace_epochs_producer" \
 "tests/test_gpu_p2p.py::test_fig3_single_block_pready" > gpurun_out/memcheck2.txt 2>&1
tail -4 gpurun_out/memcheck2.txt
PC_TIMEOUT_MS=60000 timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest -q -x tests/test_gpu_collectives.py -k "int32 or i32 or fp32 or f32" > gpurun_out/memcheck3.txt 2>&1
tail -4 gpurun_out/memcheck3.txt
