#!/bin/bash
# ncu --set full of kernels matching $KREGEX (default rowgemm) on the CFG2 driver
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"${KREGEX:-rowgemm}" -s ${SKIP:-4} -c ${COUNT:-3} -o gpurun_out/${OUT:-prof} python scripts/prof_driver.py --steps 2 ${DRIVER_ARGS} > gpurun_out/ncu_${OUT:-prof}.log 2>&1
echo "ncu rc=$?" >> gpurun_out/ncu_${OUT:-prof}.log
