#!/bin/bash
# ncu --set full of backward kernels of the CFG2 training driver (one GPU).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k regex:"${1:-rowgemm_kernel<128, 4>|wgrad_tc}" -s ${2:-0} -c ${3:-4} \
  -o gpurun_out/prof_tr python scripts/prof_driver.py --train --steps 2 > gpurun_out/prof_tr.log 2>&1
echo "rc=$?" >> gpurun_out/prof_tr.log
