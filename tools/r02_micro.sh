# microbenchmarks: TMEM read vs ex2 overlap, tcgen05.mma issue cost per N; attention kernel launch list
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tmem_ex2 tools/micro/tmem_ex2.cu && timeout 60 /tmp/tmem_ex2 | tee gpurun_out/r02_micro_tmem_ex2.txt
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Iinclude -o /tmp/mma_issue tools/micro/mma_issue.cu && timeout 120 /tmp/mma_issue | tee gpurun_out/r02_micro_mma_issue.txt
timeout 300 ncu --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,smsp__inst_executed_pipe_xu.sum,sm__cycles_active.avg --clock-control none -c 12 --csv python tools/attn_bench.py --reps 3 --b 32 > gpurun_out/r02_attn_launches.csv 2>/dev/null
python - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/r02_attn_launches.csv')) if len(r)>10]
h=rows[0]; ki=h.index('Kernel Name'); mi=h.index('Metric Name'); vi=h.index('Metric Value')
for r in rows[1:]: print(r[ki][:40], r[mi], r[vi])
PY
