# dQ GEMM on the side stream overlapped with the QKV dgrad's dK/dV columns: step tests, A/B bench;
# and the UMMA-vs-TMEM-load contention microbenchmark
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_fullsize.py -m gpu -x -q -p no:cacheprovider 2>&1 | tail -1
for v in 1 2; do
  timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/ab.json 2>gpurun_out/ab.err
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
k=d['kernels']
print('bench run $v', round(d['value'],1), round(d['ms_per_step'],2), d['clocks']['sm_mhz'], {c: round(x['seconds']/d['steps']*1e3,2) for c,x in k.items() if x['seconds']})" || tail -5 gpurun_out/ab.err
done
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Iinclude -o /tmp/mma_contention tools/micro/mma_contention.cu && timeout 120 /tmp/mma_contention | tee gpurun_out/r02_micro_mma_contention.txt
