#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 1200 python -m pytest tests -x -q -m gpu 2>&1 | tail -3 > gpurun_out/r02_pytest_gpu.txt
timeout 600 python tools/sweep.py allreduce --ranks 2,4 --algos direct --partitions 64 --max-bytes 1073741824 > gpurun_out/r02_sweep_small.jsonl 2>/dev/null
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02_smoke.txt 2>&1
cat gpurun_out/r02_pytest_gpu.txt; tail -1 gpurun_out/r02_smoke.txt
