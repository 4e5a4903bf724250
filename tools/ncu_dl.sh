#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bce_grad_multi -s 2 -c 1 -o gpurun_out/r02_dl_coop -f python tools/dl_coop_profile.py 8 16384 coop > gpurun_out/r02_ncu_dl.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:bce_grad_multi -s 2 -c 1 -o gpurun_out/r02_dl_serial_prod -f python tools/dl_coop_profile.py 8 16384 serial >> gpurun_out/r02_ncu_dl.log 2>&1
tail -2 gpurun_out/r02_ncu_dl.log
