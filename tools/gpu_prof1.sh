set -x
python tools/attn_bench.py --reps 20 2>&1 | tail -2
python tools/attn_bench.py --reps 20 --causal 1 2>&1 | tail -2
python tools/gemm_bench.py --reps 20 2>&1 | tail -14
timeout 600 python bench.py --no-cpu-baseline --steps 5 --warmup 3 > gpurun_out/bench_attnsplit.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/bench_attnsplit.json'));print(d['value'], json.dumps(d['kernels']), d['attention'], d['roofline']['achieved'])"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attn_ -c 2 -o gpurun_out/ncu_attn python tools/attn_bench.py --reps 1 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tc2 -c 12 -o gpurun_out/ncu_gemm python tools/gemm_bench.py --reps 1 > /dev/null 2>&1
ls -la gpurun_out
