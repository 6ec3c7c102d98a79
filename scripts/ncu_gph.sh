#!/bin/bash
# ncu --set full of the Graphormer attention kernel (and the decoder kernels) on CFG2.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on \
  -k regex:"${NCU_K:-gph_attn}" -s ${NCU_S:-2} -c ${NCU_C:-1} -o gpurun_out/prof_gph \
  python scripts/prof_driver.py --steps 2 --graphormer 2 ${PROF_ARGS} > gpurun_out/prof_gph.log 2>&1
echo "rc=$?" >> gpurun_out/prof_gph.log
