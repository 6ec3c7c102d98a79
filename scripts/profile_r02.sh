#!/bin/bash
# Round-2 profiling on one GPU: (1) the launch list of the bench's headline (CFG3 FP32 training
# step) under ncu --metrics gpu__time_duration.sum,dram bytes; (2) ncu --set full of one CFG3
# training step's kernels; (3) CFG2 inference kernels.  Summaries -> gpurun_out/profiles_new.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out/profiles_new
timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
  --clock-control none -c 500 --csv --log-file gpurun_out/launches.csv \
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
PROFILES_OUT=gpurun_out/profiles_new python scripts/ncu_summary.py ${TAG:-r02} gpurun_out/launches.csv \
  "gpurun_out/prof_cfg3.ncu-rep:CFG3 FP32 training step (scripts/prof_driver.py --train --cfg3):traffic_cfg3.json" \
  "gpurun_out/prof_cfg2.ncu-rep:CFG2 FP32 inference (scripts/prof_driver.py):traffic.json" > gpurun_out/summary.log 2>&1
for r in cfg3 cfg2; do
  python scripts/ncu_stalls.py gpurun_out/prof_$r.ncu-rep "wgrad_tc|node_bwd|gate_bwd|rowgemm_kernel<128, 3>|gather_segsum" 30 > gpurun_out/profiles_new/${TAG:-r02}_${r}_stalls.txt 2>&1
done
rm -f gpurun_out/prof_cfg3.ncu-rep gpurun_out/prof_cfg2.ncu-rep
