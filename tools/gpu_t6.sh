timeout 900 python -m pytest tests/test_gpu_kernels.py -x -q -k gemm 2>&1 | tail -2
GEMM_BENCH_TOKENS=16384 python tools/gemm_bench.py --graph --only out_wgrad 2>&1 | tail -2
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench exit $?"
python -c "import json;d=json.load(open('gpurun_out/bench.json'));print('cfg2', d['value'], d['roofline']['frac'], d['step_roofline']['frac_strict'], {k:round(v['seconds']/d['steps']*1e3,2) for k,v in d['kernels'].items()})"
