set -x
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 python tools/gemm_bench.py --graph > gpurun_out/gb.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python tools/profile_step.py --layers 2 --steps 2 > gpurun_out/prof_step.log 2>&1
for k in ln_bwd_v attn_bwd_persistent attn_fwd_kernel colsum_partial_vec; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$k -c 1 -o gpurun_out/full_$k python tools/profile_step.py --layers 1 --steps 1 > gpurun_out/ncu_$k.log 2>&1
done
cat gpurun_out/pytest_gpu.log; cat gpurun_out/bench.json; cat gpurun_out/gb.log
