#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 600 python tools/sweep.py p2p --batched --graph --persistent --sizes 65536,1048576,16777216,67108864,268435456 --grans block,block_put --aggs none,1MiB \
  > gpurun_out/r02_c2_v8_graph_pers.jsonl 2> gpurun_out/r02_c2_v8.err
timeout 600 python tools/sweep.py p2p --batched --graph --sizes 65536,1048576,16777216,67108864,268435456 --grans block,block_put --aggs none,1MiB \
  > gpurun_out/r02_c2_v8_graph_nonpers.jsonl 2>> gpurun_out/r02_c2_v8.err
for f in gpurun_out/r02_c2_v8_graph_*.jsonl; do echo "== $f"; python - "$f" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    try: d=json.loads(l)
    except Exception: continue
    if d.get("copy") == "engine": continue
    print(d.get("bytes")>>10, d.get("mode") or (d["gran"],d["agg"],d["copy"]), round(d["us"],1), d.get("parity",""))
PY
done; tail -3 gpurun_out/r02_c2_v8.err
