#!/bin/bash
# full GPU suite, smoke, bench (N=1), DL proxy modes
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -30 > gpurun_out/r02_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02_smoke.txt 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/r02_bench.json 2> gpurun_out/r02_bench.err
timeout 600 python tools/dl_bench.py timeline,timeline_serial,pready_inline,allreduce_only,allreduce_bounded 8,4 65536 3 > gpurun_out/r02_dl_all.jsonl 2> gpurun_out/r02_dl_all.err
tail -3 gpurun_out/r02_pytest_gpu.txt; tail -2 gpurun_out/r02_smoke.txt; cut -c1-400 gpurun_out/r02_bench.json; cat gpurun_out/r02_dl_all.jsonl
