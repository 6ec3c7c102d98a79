#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"rowgemm|edge_small" -s 4 -c 4 -o gpurun_out/prof_tc python scripts/prof_driver.py --steps 2 > gpurun_out/ncu_tc.log 2>&1
timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu --no-train > gpurun_out/bench.log 2>&1
