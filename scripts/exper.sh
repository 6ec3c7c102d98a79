#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for e in 0 1 2 3 4 7; do
  echo "== exper $e" >> gpurun_out/exper.log
  OCCU_TC_EXPER=$e timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-train 2>&1 | python scripts/show_bench.py /dev/stdin | grep kernels >> gpurun_out/exper.log
done
