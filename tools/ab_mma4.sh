# round 1: kernel tests + GEMM set after the four-UMMA issue change
timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q > gpurun_out/t_kernels.log 2>&1; echo "kernel tests $?"; tail -2 gpurun_out/t_kernels.log
timeout 300 python tools/gemm_bench.py --reps 20 --graph > gpurun_out/gb_mma4.jsonl 2>&1
python -c "
import json
r=[json.loads(l) for l in open('gpurun_out/gb_mma4.jsonl') if l.startswith('{')]
print(' '.join('%s:%.1f'%(x['gemm'],x['us']) for x in r if 'us' in x)); print('total_us %.1f'%sum(x['us'] for x in r if 'us' in x))"
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_mma4.json 2>gpurun_out/bench_mma4.err
python -c "
import json
d=json.loads(open('gpurun_out/bench_mma4.json').read().strip().splitlines()[-1]); print('bench', d['value'], d['ms_per_step'], d['roofline']['frac'], d['clocks'])"
