#!/bin/bash
# Round-2 (late) profiling on one GPU, after the CFG1 tensor-core rewrite and the sign-bit /
# fused-dW_e backward changes: (1) the launch list of the bench's default headline command;
# (2) ncu --set full of one CFG3 FP32 training step; (3) the CFG1 single-CTA kernel.
# Summaries -> gpurun_out/profiles_new.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out/profiles_new
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 500 --csv \
  --log-file gpurun_out/launches.csv \
  python bench.py --steps 3 --warmup 3 --sections '' --no-cpu --no-e2e > gpurun_out/launches_bench.log 2>&1
echo "launches rc=$?" >> gpurun_out/launches_bench.log
timeout 1800 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -s ${SKIP3:-90} -c ${COUNT3:-90} -o gpurun_out/prof_cfg3 \
  python scripts/prof_driver.py --train --cfg3 --steps 3 > gpurun_out/prof_cfg3.log 2>&1
echo "cfg3 rc=$?" >> gpurun_out/prof_cfg3.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:small_forward -s 3 -c 1 \
  -o gpurun_out/prof_cfg1 python scripts/probes/cfg1_probe.py > gpurun_out/prof_cfg1.log 2>&1
echo "cfg1 rc=$?" >> gpurun_out/prof_cfg1.log
PROFILES_OUT=gpurun_out/profiles_new python scripts/ncu_summary.py ${TAG:-r02c} gpurun_out/launches.csv \
  "gpurun_out/prof_cfg3.ncu-rep:CFG3 FP32 training step (scripts/prof_driver.py --train --cfg3):traffic_cfg3.json" \
  "gpurun_out/prof_cfg1.ncu-rep:CFG1 single-CTA forward (scripts/probes/cfg1_probe.py):traffic_cfg1.json" \
  > gpurun_out/summary.log 2>&1
python scripts/ncu_stalls.py gpurun_out/prof_cfg3.ncu-rep "wgrad_tc|node_bwd|gate_bwd|rowgemm_kernel<128, 3>|rowgemm_kernel<128, 5>" 30 > gpurun_out/profiles_new/${TAG:-r02c}_cfg3_stalls.txt 2>&1
rm -f gpurun_out/prof_cfg3.ncu-rep gpurun_out/prof_cfg1.ncu-rep
