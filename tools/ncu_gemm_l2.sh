# ncu --set full of the CTA-pair GEMM on two cfg2 shapes (QKV forward: K-major operands; FC1 weight
# gradient: MN-major A and B, K = 16384 tokens) for the L2 / TMA-throughput evidence of DESIGN §4.
#   gpurun --timeout 1200 -- 'bash tools/ncu_gemm_l2.sh'
set -x
mkdir -p gpurun_out
for s in qkv_fwd fc1_wgrad; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tc2 -c 1 -s 3 \
    -o gpurun_out/ncu_gemm_$s -f python tools/gemm_bench.py --only $s --reps 3 > gpurun_out/ncu_gemm_$s.log 2>&1
  echo "ncu $s exit $?"
  python tools/ncu_summary.py gpurun_out/ncu_gemm_$s.ncu-rep --grep \
    'lts__t_bytes|lts__throughput|lts__t_sector_hit_rate|lts__d|l1tex__m_xbar2l1tex|gpu__compute_memory_throughput|smsp__pcsamp|dram__throughput|sm__inst_executed_pipe_tma|tma' \
    > gpurun_out/ncu_gemm_$s.txt 2>&1
  head -60 gpurun_out/ncu_gemm_$s.txt
done
# the same shapes timed without the profiler (CUDA events, warm)
timeout 300 python tools/gemm_bench.py --reps 20 --cublas > gpurun_out/gemm_bench_cfg2.jsonl 2>&1
cat gpurun_out/gemm_bench_cfg2.jsonl
