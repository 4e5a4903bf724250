#!/bin/bash
# DL proxy: one-launch interleaved producers — serial vs INLINE fold vs cooperative INLINE fold (R36) vs engine
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_dl.py tests/test_gpu_inline_allreduce.py -x -q -m gpu 2>&1 | tail -5 > gpurun_out/r02_dl_multi_pytest.txt
timeout 900 python tools/dl_bench.py serial,serial_multi,pready_inline_multi,pready_coop_multi,pready 8,4,2 4096,16384,65536 3 \
  > gpurun_out/r02_dl_multi.jsonl 2> gpurun_out/r02_dl_multi.err
cat gpurun_out/r02_dl_multi_pytest.txt; python - <<'PY'
import json
for l in open("gpurun_out/r02_dl_multi.jsonl"):
    d=json.loads(l); print(d.get("P"), d.get("partition_bytes"), d.get("mode"), round(d.get("ms_per_step",0),3), d.get("error",""))
PY
tail -3 gpurun_out/r02_dl_multi.err
