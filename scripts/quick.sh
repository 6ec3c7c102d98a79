#!/bin/bash
# quick GPU iteration: tc parity subset + short bench
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "${PYTEST_K:-tcgen05 or cfg or determinism or batching or agree}" > gpurun_out/pytest_quick.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_quick.log
timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu ${BENCH_ARGS} > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
