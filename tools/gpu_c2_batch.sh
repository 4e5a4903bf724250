#!/bin/bash
# batched release of the persistent register Kernel Copy: parity, then the C2 sweep per batch size
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_p2p.py -x -q -m gpu -k "put_batched or persistent or producer_shapes" 2>&1 | tail -3 > gpurun_out/r02_c2_batch_pytest.txt
for b in 1 2 4 8 16; do
  PCAPP_PUT_BATCH=$b timeout 600 python tools/sweep.py p2p --batched --persistent --sizes 1048576,16777216,67108864,268435456 --grans block_put --aggs none \
    > gpurun_out/r02_c2_batch$b.jsonl 2>> gpurun_out/r02_c2_batch.err
  PCAPP_PUT_BATCH=$b timeout 600 python tools/sweep.py p2p --batched --graph --persistent --sizes 16777216,268435456 --grans block_put --aggs none \
    > gpurun_out/r02_c2_batch${b}_graph.jsonl 2>> gpurun_out/r02_c2_batch.err
done
cat gpurun_out/r02_c2_batch_pytest.txt
for f in gpurun_out/r02_c2_batch*.jsonl; do echo "== $f"; python - "$f" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    try: d=json.loads(l)
    except Exception: continue
    if d.get("copy") == "engine": continue
    print(d.get("bytes")>>10, d.get("mode") or (d["gran"],d["agg"],d["copy"]), round(d["us"],1), d.get("parity",""))
PY
done; tail -3 gpurun_out/r02_c2_batch.err
