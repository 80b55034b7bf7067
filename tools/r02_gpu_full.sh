# full gpu suite + default bench + kernel timeline, at HEAD
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/t_all.log 2>&1; echo "all gpu tests $?"; tail -3 gpurun_out/t_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke $?"; tail -1 gpurun_out/smoke.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; echo "bench $?"
python -c "import json;d=json.loads(open('gpurun_out/bench_full.json').read().strip().splitlines()[-1]);print('bench', d['value'], d['ms_per_step'], d['roofline']['frac'], d['roofline'].get('achieved_while_running'), d['step_roofline']['frac_strict'], d['clocks'], d['e2e']['value'], d['cpu_baseline'])"
cd tools && timeout 600 python ktimeline.py --out ../gpurun_out/ktl_head.json > ../gpurun_out/ktl_head.txt 2>&1; echo "ktl $?"; cd ..
