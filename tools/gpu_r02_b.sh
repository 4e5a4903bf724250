#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_fullsize_jacobi.py "tests/test_gpu_p2p.py::test_c2_block_256mib" -x -q 2>&1 | tail -8 > gpurun_out/r02_fullsize_pytest.txt
timeout 900 python tools/sweep.py allreduce --ranks 8,4 --algos direct,ring --partitions 64 --max-bytes 268435456 > gpurun_out/r02_sweep_ar.jsonl 2> gpurun_out/r02_sweep_ar.err
timeout 600 python tools/sweep.py coll --ranks 8 --max-bytes 268435456 > gpurun_out/r02_sweep_coll.jsonl 2> gpurun_out/r02_sweep_coll.err
timeout 600 python tools/sweep.py dl_tensor --ranks 8 > gpurun_out/r02_sweep_dlt.jsonl 2> gpurun_out/r02_sweep_dlt.err
cat gpurun_out/r02_fullsize_pytest.txt; tail -3 gpurun_out/r02_sweep_ar.err gpurun_out/r02_sweep_coll.err
