python tools/attn_bench.py --reps 20 | tail -1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attn_bwd -c 2 -o gpurun_out/ncu_attn_bwd python tools/attn_bench.py --reps 1 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attn_fwd -c 1 -o gpurun_out/ncu_attn_fwd16 python tools/attn_bench.py --reps 1 > /dev/null 2>&1
ls gpurun_out
