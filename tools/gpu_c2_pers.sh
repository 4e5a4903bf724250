#!/bin/bash
# C2: block / block_put Pready, both producer shapes; p2p parity first
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_p2p.py -x -q -m gpu -k "persistent or producer_shapes or c2_block" 2>&1 | tail -15 > gpurun_out/r02_c2_pytest_p2p.txt
for pers in "" "--persistent"; do
  tag=${pers:+pers}; tag=${tag:-nonpers}
  timeout 600 python tools/sweep.py p2p --sizes 65536,1048576,16777216,67108864,268435456 --grans block,block_put --aggs none,1MiB $pers \
    > gpurun_out/r02_c2_v7_$tag.jsonl 2> gpurun_out/r02_c2_v7_$tag.err
done
cat gpurun_out/r02_c2_pytest_p2p.txt
for f in gpurun_out/r02_c2_v7_*pers.jsonl; do echo "== $f"; python - "$f" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    try: d=json.loads(l)
    except Exception: continue
    print(d.get("bytes")>>20, d.get("mode") or (d["gran"],d["agg"],d["copy"]), round(d["us"],1), d.get("parity",""))
PY
done; for f in gpurun_out/r02_c2_v6*.err; do tail -n 3 $f; done
