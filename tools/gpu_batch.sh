#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_batch.py -x -q 2>&1 | tail -25 > gpurun_out/r02_batch_pytest.txt
timeout 600 python tools/sweep.py dl_tensor --ranks 8,4 --batched > gpurun_out/r02_dlt_batched.jsonl 2> gpurun_out/r02_dlt_batched.err
timeout 600 python tools/sweep.py dl --ranks 8 --algos direct > gpurun_out/r02_dl_flat.jsonl 2>> gpurun_out/r02_dlt_batched.err
tail -5 gpurun_out/r02_batch_pytest.txt; cat gpurun_out/r02_dlt_batched.jsonl gpurun_out/r02_dl_flat.jsonl; tail -3 gpurun_out/r02_dlt_batched.err
