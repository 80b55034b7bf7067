timeout 300 ncu --set full --import-source on --clock-control none -k regex:attn_bwd_persistent -c 1 -o gpurun_out/ncu_bwd2 python tools/attn_bench.py --reps 1 > /dev/null 2>&1
ls gpurun_out/
