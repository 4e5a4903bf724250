#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_inline_allreduce.py -x -q 2>&1 | tail -25 > gpurun_out/r02_inline_pytest.txt
timeout 300 python tools/dl_bench.py pready_inline,serial 8,4,2 65536,262144 3 > gpurun_out/r02_dl_inline.jsonl 2> gpurun_out/r02_dl_inline.err
cat gpurun_out/r02_inline_pytest.txt | tail -5; cat gpurun_out/r02_dl_inline.jsonl
