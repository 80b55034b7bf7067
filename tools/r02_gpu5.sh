# step, group and PP tests plus a short cfg2 bench
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_group.py tests/test_gpu_pp.py -m gpu -x -q > gpurun_out/t_step.log 2>&1; echo "tests $?"; tail -2 gpurun_out/t_step.log
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_h5.json 2> gpurun_out/bench_h5.err; echo "bench $?"
python -c "import json;d=json.loads(open('gpurun_out/bench_h5.json').read().strip().splitlines()[-1]);print('bench', d['value'], d['ms_per_step'], d['e2e'], d['clocks'])"
