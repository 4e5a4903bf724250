#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_p2p.py -x -q -m gpu -k "producer_shapes or c2_persistent or put_batched" 2>&1 | tail -2
timeout 600 python tools/sweep.py p2p --batched --graph --sizes 1048576,16777216,268435456 --grans block,block_put --aggs none > gpurun_out/r02d_c2_put_np.jsonl 2>/dev/null
python - <<'PY'
import json
for l in open("gpurun_out/r02d_c2_put_np.jsonl"):
    d=json.loads(l)
    if d.get("copy")=="engine": continue
    print(d["bytes"]>>10, d.get("mode") or (d["gran"], d["copy"]), round(d["us"],1), d.get("parity",""))
PY
