# round-2 wrap-up on one B200: LayerNorm micro-bench, the reference arm, the tuner (incumbent always
# measured), the full -m gpu suite and smoke() at HEAD
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 300 python tools/ln_bench.py > gpurun_out/r02_ln_bench.txt 2>&1; echo "ln $?"; cat gpurun_out/r02_ln_bench.txt | tail -3
SECONDS=0; timeout 1500 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/r02_final_ref.json 2> gpurun_out/r02_final_ref.err; echo "ref $? wall ${SECONDS}s"; tail -1 gpurun_out/r02_final_ref.json
timeout 1500 python bench.py --tune --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r02_final_cfg2_tuned.json 2> gpurun_out/r02_final_cfg2_tuned.err; echo "tune $?"
python -c "
import json
d=json.loads(open('gpurun_out/r02_final_cfg2_tuned.json').read().strip().splitlines()[-1])
print(d['value'], json.dumps(d['config'].get('tuning'))[:1500])"
timeout 2400 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/r02_gpu_tests_head_b.txt 2>&1; echo "tests $?"; tail -3 gpurun_out/r02_gpu_tests_head_b.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02_smoke.txt 2>&1; echo "smoke $?"; tail -2 gpurun_out/r02_smoke.txt
