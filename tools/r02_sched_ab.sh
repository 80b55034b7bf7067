# attention variants still correct; step scheduling A/B: side stream for weight gradients, stream priority
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -p no:cacheprovider -k "fused_attention" 2>&1 | tail -1
HARMONY_ATTN_BWD_ALT=1 HARMONY_ATTN_POLY=12 timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -p no:cacheprovider -k "fused_attention" 2>&1 | tail -1
for c in 0 1; do timeout 120 python tools/attn_bench.py --reps 20 --causal $c --b 32 2>&1 | grep attn_fwd | sed "s/^/causal$c /"; done
for v in "" "HARMONY_NO_SIDE=1" "HARMONY_PRIO=0"; do
  env $v timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/ab.json 2>/dev/null
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
print('$v', 'samples/s', round(d['value'],1), 'ms', round(d['ms_per_step'],2), 'clk', d['clocks']['sm_mhz'])"
done
