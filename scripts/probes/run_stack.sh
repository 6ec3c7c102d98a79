timeout 900 python -m pytest tests/test_gpu_graphormer.py tests/test_gpu_decoder.py -x -q 2>&1 | tail -2
timeout 600 python bench.py --steps 5 --warmup 3 --sections paper_stack_train --no-cpu --no-e2e 2>&1 | grep "\[bench\]" | tail -1
python -c "
import json; d=json.load(open('gpurun_out/bench_details.json'))['sections']['cfg2_paper_stack_train_f32']
k=d['kernel_ms_per_step']; print(d['ms_per_step'], {n:round(v,3) for n,v in sorted(k.items(), key=lambda x:-x[1])[:6]})"
