#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_allreduce.py tests/test_gpu_fullsize.py tests/test_gpu_multiproc.py -x -q 2>&1 | tail -3 > gpurun_out/r02_maxp_pytest.txt
timeout 900 python tools/sweep.py allreduce --ranks 2,4,8 --algos direct --partitions 64 --max-bytes 1073741824 > gpurun_out/r02_sweep_maxp.jsonl 2> gpurun_out/r02_sweep_maxp.err
cat gpurun_out/r02_maxp_pytest.txt
