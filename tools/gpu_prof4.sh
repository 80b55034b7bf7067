timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/traffic_m2.csv python tools/profile_step.py --layers 2 --steps 2 > /dev/null 2>&1
python tools/traffic_summary.py gpurun_out/traffic_m2.csv --last 420 > gpurun_out/traffic_cfg2_m2.json
python tools/launch_shares.py gpurun_out/traffic_m2.csv --last 420 > gpurun_out/launch_shares_m2.txt
head -25 gpurun_out/launch_shares_m2.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tc2 -c 1 -o gpurun_out/ncu_full_qkv_fwd_m2 env GEMM_BENCH_TOKENS=16384 python tools/gemm_bench.py --reps 1 --only qkv_fwd > /dev/null 2>&1
ls gpurun_out | grep -E "m2"
