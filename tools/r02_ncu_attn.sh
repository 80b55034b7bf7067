# ncu --set full of the fused attention forward and backward at the cfg2 shape (b=32, S=512, h=16)
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:attn_bwd_persistent -c 1 -o gpurun_out/r02_ncu_full_attn_bwd -f python tools/attn_bench.py --reps 1 --b 32 > gpurun_out/ncu_attn.log 2>&1; echo "ncu $?"
