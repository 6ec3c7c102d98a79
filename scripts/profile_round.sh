#!/bin/bash
# Round profiling (one GPU): launch list of the bench command + ncu --set full of
# the hot kernels; summarised into profiles/ by scripts/summarize_ncu.py (run here).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
  --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 3 --warmup 3 --no-cpu > gpurun_out/launches_bench.log 2>&1
echo "launches rc=$?" >> gpurun_out/launches_bench.log
timeout 900 ncu --set full --clock-control none --import-source on \
  -k regex:"rowgemm|gather_segsum|edge_small" -s 7 -c 7 -o gpurun_out/prof_full \
  python scripts/prof_driver.py --steps 2 > gpurun_out/prof_full.log 2>&1
echo "full rc=$?" >> gpurun_out/prof_full.log
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k regex:"rowgemm_kernel<\(int\)128, \(int\)[45]>|wgrad_tc|split_reduce|node_bwd" -s 12 -c 8 -o gpurun_out/prof_train \
  python scripts/prof_driver.py --steps 3 --train > gpurun_out/prof_train.log 2>&1
echo "train rc=$?" >> gpurun_out/prof_train.log
timeout 900 ncu --set full --clock-control none --import-source on \
  -k regex:"rowgemm|gather_segsum|edge_small" -s 7 -c 7 -o gpurun_out/prof_bf16 \
  python scripts/prof_driver.py --steps 2 --bf16 > gpurun_out/prof_bf16.log 2>&1
echo "bf16 rc=$?" >> gpurun_out/prof_bf16.log
timeout 900 ncu --set full --clock-control none --import-source on \
  -k regex:"gph_|set_decoder|synth" -s 10 -c 9 -o gpurun_out/prof_next \
  python scripts/prof_driver.py --steps 2 --graphormer 2 --decoder --synth > gpurun_out/prof_next.log 2>&1
echo "next rc=$?" >> gpurun_out/prof_next.log
# summarise on the box (the .ncu-rep files are too big to bring back whole)
PROFILES_OUT=gpurun_out/profiles_new python scripts/summarize_ncu.py ${TAG:-r01} > gpurun_out/summarize.log 2>&1
for f in gpurun_out/prof_*.ncu-rep; do
  python scripts/ncu_stalls.py "$f" "gph_attn|gather_segsum|set_decoder|synth" 30 > "${f%.ncu-rep}_stalls.txt" 2>&1
done
du -sh gpurun_out/* > gpurun_out/sizes.txt
rm -f gpurun_out/prof_full.ncu-rep gpurun_out/prof_train.ncu-rep gpurun_out/prof_bf16.ncu-rep
