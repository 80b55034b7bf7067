# round 2, second GPU pass: group (N>1 loopback) tests + split-GEMM K-split, sanitizer on the group,
# kernel timelines of the cfg2 step (policies 2, 3), bench policy 3, ncu launch list of a 2-layer step.
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_group.py tests/test_gpu_split_gemm.py -m gpu -x -q -s -k "group or loopback or full_check" > gpurun_out/t_group.log 2>&1; echo "group tests $?"; tail -4 gpurun_out/t_group.log
HARMONY_NO_GRAPH=1 timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_step.py group > gpurun_out/memcheck_group.log 2>&1; echo "memcheck group $?"; tail -3 gpurun_out/memcheck_group.log
HARMONY_NO_GRAPH=1 timeout 900 compute-sanitizer --tool synccheck --print-limit 20 python tools/sanitize_step.py cfg1 group > gpurun_out/synccheck.log 2>&1; echo "synccheck $?"; tail -3 gpurun_out/synccheck.log
cd tools && timeout 600 python ktimeline.py --out ../gpurun_out/ktl_p2.json > ../gpurun_out/ktl_p2.txt 2>&1; echo "ktl p2 $?"; cd ..
cd tools && timeout 600 python ktimeline.py --stash-policy 3 --out ../gpurun_out/ktl_p3.json > ../gpurun_out/ktl_p3.txt 2>&1; echo "ktl p3 $?"; cd ..
head -60 gpurun_out/ktl_p2.txt
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_p2.json 2> gpurun_out/bench_p2.err; echo "bench p2 $?"
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --stash-policy 3 > gpurun_out/bench_p3.json 2> gpurun_out/bench_p3.err; echo "bench p3 $?"
for f in p2 p3; do python -c "import json;d=json.loads(open('gpurun_out/bench_$f.json').read().strip().splitlines()[-1]);print('$f', d['value'], d['ms_per_step'], d['roofline']['frac'], d['roofline'].get('achieved_while_running'), d['step_roofline']['frac_strict'], d['clocks'])"; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_launches_cfg2_2layers.csv python tools/profile_step.py --layers 2 --steps 2 > gpurun_out/ncu_step.log 2>&1; echo "ncu list $?"
python tools/launch_shares.py gpurun_out/r02_launches_cfg2_2layers.csv | head -30
