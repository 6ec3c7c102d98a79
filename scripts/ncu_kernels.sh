#!/bin/bash
# ncu --set full of selected kernels of the CFG2 inference driver (one GPU).
# usage: ncu_kernels.sh OUTNAME KERNEL_REGEX [SKIP] [COUNT] [driver args...]
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
out=$1; kre=$2; skip=${3:-0}; cnt=${4:-4}; shift 4
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"$kre" -s $skip -c $cnt \
  -o gpurun_out/$out python scripts/prof_driver.py "$@" > gpurun_out/$out.log 2>&1
echo "rc=$?" >> gpurun_out/$out.log
