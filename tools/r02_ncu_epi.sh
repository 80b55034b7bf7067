# ncu --set full of the specialised FC1-forward / FC2-dgrad GEMM kernels
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
for k in fc1_fwd fc2_dgrad; do
timeout 600 ncu --set full --import-source on --clock-control none -k regex:gemm_tc2 -c 1 -s 3 -o gpurun_out/r02_ncu_spec_$k -f python tools/gemm_bench.py --only $k --reps 3 > gpurun_out/ncu_$k.log 2>&1; echo "ncu $k $?"
done
