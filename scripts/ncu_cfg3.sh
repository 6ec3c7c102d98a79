#!/bin/bash
# ncu --set full of CFG3 training-step kernels matching $1 (demangled names), one GPU.
#   scripts/ncu_cfg3.sh '<kernel regex>' [skip] [count] [out]
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
OUT=${4:-cfg3}
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k regex:"${1:-rowgemm_kernel<128, 5>}" -s ${2:-0} -c ${3:-1} \
  -o gpurun_out/$OUT python scripts/prof_driver.py --train --cfg3 --steps 2 > gpurun_out/$OUT.log 2>&1
echo "rc=$?" >> gpurun_out/$OUT.log
python scripts/ncu_stalls.py gpurun_out/$OUT.ncu-rep "${1:-rowgemm_kernel<128, 5>}" 40 > gpurun_out/${OUT}_stalls.txt 2>&1
