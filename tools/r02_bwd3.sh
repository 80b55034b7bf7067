# attention backward with three score buffers (P^T in shared memory): kernel tests, ncu durations, bench
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -p no:cacheprovider -k "fused_attention" 2>&1 | tail -1
HARMONY_ATTN_BWD_ALT=1 timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -p no:cacheprovider -k "fused_attention_backward" 2>&1 | tail -1
for c in 0 1; do
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:attn_bwd_persistent -c 3 --csv python tools/attn_bench.py --reps 3 --b 32 --causal $c 2>/dev/null | grep -E "gpu__time" | awk -F'","' -v c=$c '{print "causal" c, $(NF-2), $NF}'
done
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/ab.json 2>gpurun_out/ab.err
python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
k=d['kernels']
print('bench', round(d['value'],1), round(d['ms_per_step'],2), d['clocks']['sm_mhz'], d['attention'], {c: round(x['seconds']/d['steps']*1e3,2) for c,x in k.items() if x['seconds']})" || tail -5 gpurun_out/ab.err
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_fullsize.py -m gpu -x -q -p no:cacheprovider 2>&1 | tail -1
