# A/B of the persistent GEMM's tile raster width (HARMONY_GEMM_GROUP_M): cfg2 GEMM shapes through
# hk_gemm (CUDA events, graph replay), then the default bench at each candidate.
#   gpurun --timeout 1500 -- 'bash tools/ab_group_m.sh'
mkdir -p gpurun_out
for g in 1 2 4 8 16 64; do
  echo "== group_m $g"
  HARMONY_GEMM_GROUP_M=$g timeout 300 python tools/gemm_bench.py --reps 20 --graph 2>&1 | \
    python -c "
import json, sys
r = [json.loads(l) for l in sys.stdin if l.startswith('{')]
print(' '.join('%s:%.1f' % (x['gemm'], x['us']) for x in r if 'us' in x))
print('total_us %.1f' % sum(x['us'] for x in r if 'us' in x))"
done 2>&1 | tee gpurun_out/ab_group_m.txt
for g in 8 ${AB_BENCH:-4 16}; do
  HARMONY_GEMM_GROUP_M=$g timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_g$g.json 2> gpurun_out/bench_g$g.err
  python -c "
import json
d = json.loads(open('gpurun_out/bench_g$g.json').read().strip().splitlines()[-1])
print('bench group_m $g', round(d['value'], 1), round(d['ms_per_step'], 2), d['clocks'])" | tee -a gpurun_out/ab_group_m.txt
done
