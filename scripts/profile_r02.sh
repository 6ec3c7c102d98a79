#!/bin/bash
# Round-2 profiling on one GPU: (1) the launch list of the bench's default command (headline
# CFG3 FP32 training step; the recipe's --metrics gpu__time_duration.sum --clock-control none
# pass); (2) ncu --set full of one CFG3 training step's kernels; (3) CFG2 inference kernels;
# (4) the d = 256 CTA-pair kernels (CFG2-paper, L = 1).  Summaries -> gpurun_out/profiles_new.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out/profiles_new
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 500 --csv \
  --log-file gpurun_out/launches.csv \
  python bench.py --steps 3 --warmup 3 --sections '' --no-cpu --no-e2e > gpurun_out/launches_bench.log 2>&1
echo "launches rc=$?" >> gpurun_out/launches_bench.log
# one CFG3 training step = the second prof_driver step (the first builds images / allocates)
timeout 1800 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -s ${SKIP3:-90} -c ${COUNT3:-90} -o gpurun_out/prof_cfg3 \
  python scripts/prof_driver.py --train --cfg3 --steps 3 > gpurun_out/prof_cfg3.log 2>&1
echo "cfg3 rc=$?" >> gpurun_out/prof_cfg3.log
timeout 900 ncu --set full --clock-control none --import-source on \
  -k regex:"rowgemm|gather_segsum|edge_small|readout" -s 12 -c 12 -o gpurun_out/prof_cfg2 \
  python scripts/prof_driver.py --steps 3 > gpurun_out/prof_cfg2.log 2>&1
echo "cfg2 rc=$?" >> gpurun_out/prof_cfg2.log
timeout 900 ncu --set full --clock-control none --import-source on \
  -k regex:"rowgemm_pair|row_exp|gather_segsum|edge_small|readout" -s 6 -c 6 -o gpurun_out/prof_d256 \
  python scripts/prof_driver.py --d 256 --L 1 --steps 3 > gpurun_out/prof_d256.log 2>&1
echo "d256 rc=$?" >> gpurun_out/prof_d256.log
PROFILES_OUT=gpurun_out/profiles_new python scripts/ncu_summary.py ${TAG:-r02} gpurun_out/launches.csv \
  "gpurun_out/prof_cfg3.ncu-rep:CFG3 FP32 training step (scripts/prof_driver.py --train --cfg3):traffic_cfg3.json" \
  "gpurun_out/prof_cfg2.ncu-rep:CFG2 FP32 inference (scripts/prof_driver.py):traffic.json" \
  "gpurun_out/prof_d256.ncu-rep:CFG2-paper FP32 inference, L = 1, d = 256 (scripts/prof_driver.py --d 256 --L 1):traffic_d256.json" \
  > gpurun_out/summary.log 2>&1
for r in cfg3 cfg2; do
  python scripts/ncu_stalls.py gpurun_out/prof_$r.ncu-rep "wgrad_tc|node_bwd|gate_bwd|rowgemm_kernel<128, 3>|gather_segsum" 30 > gpurun_out/profiles_new/${TAG:-r02}_${r}_stalls.txt 2>&1
done
python scripts/probes/pair_stalls.py gpurun_out/prof_d256.ncu-rep "(int)2" 40 > gpurun_out/profiles_new/${TAG:-r02}_d256_gate_stalls.txt 2>&1
rm -f gpurun_out/prof_cfg3.ncu-rep gpurun_out/prof_cfg2.ncu-rep gpurun_out/prof_d256.ncu-rep
