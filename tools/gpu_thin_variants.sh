#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out; rm -f gpurun_out/r02_thin_variants.jsonl
for lib in libpc libpc_thin_fv2 libpc_thin_bulk1k libpc_thin_bulk1k3; do
  for f in 0.5 1.0; do
    PC_LIB=paper_conf_sc_temucinslsga24_b200/$lib.so PC_OVERLAP_FRAC=$f timeout 300 python tools/dl_bench.py timeline,allreduce_bounded 8 16384 3 \
      | sed "s/^{/{\"lib\": \"$lib\", \"frac\": $f, /" >> gpurun_out/r02_thin_variants.jsonl 2>> gpurun_out/r02_thin_variants.err
  done
done
PC_LIB=paper_conf_sc_temucinslsga24_b200/libpc.so timeout 300 python tools/dl_bench.py timeline_serial,allreduce_only 8 16384 3 >> gpurun_out/r02_thin_variants.jsonl 2>> gpurun_out/r02_thin_variants.err
cat gpurun_out/r02_thin_variants.jsonl | cut -c1-200; tail -3 gpurun_out/r02_thin_variants.err
