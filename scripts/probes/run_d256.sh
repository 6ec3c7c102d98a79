timeout 600 python -m pytest tests/test_gpu_d256.py -x -q > gpurun_out/t256.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 --sections cfg2_paper,micro --no-cpu --no-e2e > gpurun_out/b256.out 2> gpurun_out/b256.err; echo rc=$?
grep "\[bench\]" gpurun_out/b256.err | tail -8
python - <<'PY'
import json
d=json.load(open("gpurun_out/bench_details.json"))["sections"]
x=d.get("cfg2_paper_f32",{})
print(x.get("ms_per_step"), x.get("gate_tensor_roofline",{}).get("frac"))
for k,v in x.get("kernels",{}).items(): print(k, round(v["ms_per_step"]*1e3,1), "us", round(v.get("frac_of_measured_hbm") or 0,3))
PY
if [ -n "$PROF" ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"rowgemm_pair" -s 3 -c 3 -o gpurun_out/prof_pair python scripts/prof_driver.py --d 256 --L 1 --steps 3 > gpurun_out/prof_pair.log 2>&1
python scripts/probes/pair_stalls.py gpurun_out/prof_pair.ncu-rep "(int)2" 30
python scripts/ncu_stalls.py gpurun_out/prof_pair.ncu-rep 2>&1 | head -4
fi
tail -3 gpurun_out/t256.log
