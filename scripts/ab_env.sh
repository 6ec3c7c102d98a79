#!/bin/bash
# A/B runtime variants on one GPU: each argument is an env assignment list
# ("OCCU_GATHER_V=1 OCCU_GATHER_BPS=4"); runs a short inference bench per variant.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
: > gpurun_out/ab.log
for v in "$@"; do
  echo "=== $v" >> gpurun_out/ab.log
  env $v timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu --no-train ${BENCH_ARGS} >> gpurun_out/ab.log 2>&1
done
