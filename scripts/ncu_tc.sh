#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"gate_agg|node_tc|edge_tc" -s 3 -c 3 -o gpurun_out/prof_tc python scripts/prof_driver.py --steps 2 > gpurun_out/ncu_tc.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"gather_segsum" -s 3 -c 1 -o gpurun_out/prof_gather python scripts/prof_driver.py --steps 2 --path 1 > gpurun_out/ncu_gather.log 2>&1
ls -la gpurun_out
