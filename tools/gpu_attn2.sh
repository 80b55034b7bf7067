timeout 300 ncu --set full --import-source on --clock-control none -k regex:attn_fwd -c 1 -o gpurun_out/ncu_fwd1p python tools/attn_bench.py --reps 1 > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:attn_fwd -c 1 -o gpurun_out/ncu_fwd1p_causal python tools/attn_bench.py --reps 1 --causal 1 > /dev/null 2>&1
ls gpurun_out | grep fwd1p
