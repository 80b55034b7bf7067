# GEMM: our fused-epilogue kernels vs cuBLAS plain and vs the library-equivalent fused op; ncu full
# (source-level) of the FC1 forward (GeLU two-output epilogue) and the FC2 dgrad (GeLU' epilogue)
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 300 python tools/gemm_bench.py --cublas --reps 20 > gpurun_out/r02_gemm_vs_cublas_fused.jsonl 2>&1; echo "bench $?"
cat gpurun_out/r02_gemm_vs_cublas_fused.jsonl | python -c "
import sys,json
for l in sys.stdin:
  try: d=json.loads(l)
  except Exception: print(l.strip()); continue
  print(d['gemm'], round(d.get('us',0),1), round(d.get('cublas_us',0),1), round(d.get('cublas_fused_us',0),1), round(d.get('vs_cublas_fused',0),3))"
for k in fc1_fwd fc2_dgrad; do
timeout 600 ncu --set full --import-source on --clock-control none -k regex:gemm_tc2 -c 1 -s 3 -o gpurun_out/r02_ncu_full_gemm_$k -f python tools/gemm_bench.py --only $k --reps 3 > /dev/null 2>&1; echo "ncu $k $?"
done
