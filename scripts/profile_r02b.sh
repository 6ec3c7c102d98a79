#!/bin/bash
# Round-2 follow-up captures: the paper-stack training step's attention backward (mma.sync TF32
# split) and the d = 256 BF16 CTA-pair kernels.  Summaries -> gpurun_out/profiles_new.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out/profiles_new
timeout 900 ncu --set full --clock-control none --import-source on \
  -k regex:"attn_bwd|gph_attn|dec_pool_bwd|ln_bwd" -s 8 -c 8 -o gpurun_out/prof_stack \
  python scripts/prof_driver.py --train --graphormer 2 --decoder --steps 2 > gpurun_out/prof_stack.log 2>&1
echo "stack rc=$?" >> gpurun_out/prof_stack.log
timeout 900 ncu --set full --clock-control none --import-source on \
  -k regex:"rowgemm_pair|gather_segsum|edge_small|readout" -s 5 -c 5 -o gpurun_out/prof_d256b \
  python scripts/prof_driver.py --d 256 --L 1 --bf16 --steps 3 > gpurun_out/prof_d256b.log 2>&1
echo "d256b rc=$?" >> gpurun_out/prof_d256b.log
PROFILES_OUT=gpurun_out/profiles_new python scripts/ncu_summary.py ${TAG:-r02b} none \
  "gpurun_out/prof_stack.ncu-rep:CFG2 paper-stack FP32 training step, attention / decoder / LN backward (scripts/prof_driver.py --train --graphormer 2 --decoder):traffic_stack_train.json" \
  "gpurun_out/prof_d256b.ncu-rep:CFG2-paper BF16 inference, L = 1, d = 256 (scripts/prof_driver.py --d 256 --L 1 --bf16):traffic_d256_bf16.json" \
  > gpurun_out/summary_b.log 2>&1
python scripts/probes/pair_stalls.py gpurun_out/prof_stack.ncu-rep "attn_bwd_q_mma" 30 > gpurun_out/profiles_new/r02b_attn_bwd_stalls.txt 2>&1
python scripts/probes/pair_stalls.py gpurun_out/prof_stack.ncu-rep "attn_bwd_kv_mma" 30 >> gpurun_out/profiles_new/r02b_attn_bwd_stalls.txt 2>&1
python scripts/probes/pair_stalls.py gpurun_out/prof_d256b.ncu-rep "rowgemm_pair_kernel<(int)2" 30 > gpurun_out/profiles_new/r02b_d256_gate_stalls.txt 2>&1
rm -f gpurun_out/prof_stack.ncu-rep gpurun_out/prof_d256b.ncu-rep
