# fusions (cast+colsum of dY, db_o in the LN2 backward): kernel + step tests; bench A/B side stream
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_step.py tests/test_gpu_kernels.py tests/test_gpu_group.py -m gpu -x -q > gpurun_out/t_step.log 2>&1; echo "step tests $?"; tail -3 gpurun_out/t_step.log
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_side.json 2> gpurun_out/bench_side.err; echo "bench side $?"
HARMONY_NO_SIDE=1 timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_noside.json 2> gpurun_out/bench_noside.err; echo "bench noside $?"
for f in side noside; do python -c "import json;d=json.loads(open('gpurun_out/bench_$f.json').read().strip().splitlines()[-1]);print('$f', d['value'], d['ms_per_step'], d['roofline']['frac'], d['roofline'].get('achieved_while_running'), d['step_roofline']['frac_strict'], d['clocks'])"; done
cd tools && HARMONY_NO_SIDE=1 timeout 600 python ktimeline.py --out ../gpurun_out/ktl_noside.json > ../gpurun_out/ktl_noside.txt 2>&1; echo "ktl noside $?"; cd ..
