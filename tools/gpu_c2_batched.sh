#!/bin/bash
# C2 with batched control (pc_epoch_all + pc_waitall_on_stream), both producer shapes
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for pers in "" "--persistent"; do
  tag=${pers:+pers}; tag=${tag:-nonpers}
  timeout 600 python tools/sweep.py p2p --batched --sizes 65536,1048576,16777216,67108864,268435456 --grans block,block_put --aggs none,1MiB $pers \
    > gpurun_out/r02_c2_v7b_$tag.jsonl 2> gpurun_out/r02_c2_v7b_$tag.err
done
for f in gpurun_out/r02_c2_v7b_*pers.jsonl; do echo "== $f"; python - "$f" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    try: d=json.loads(l)
    except Exception: continue
    print(d.get("bytes")>>10, d.get("mode") or (d["gran"],d["agg"],d["copy"]), round(d["us"],1), d.get("parity",""))
PY
done; for f in gpurun_out/r02_c2_v7b*.err; do tail -n 3 $f; done
