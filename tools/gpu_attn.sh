timeout 600 python -m pytest tests/test_gpu_kernels.py -x -q -k "attention" 2>&1 | tail -2
python tools/attn_bench.py --reps 20 | tail -1
python tools/attn_bench.py --reps 20 --causal 1 | tail -1
python tools/attn_bench.py --reps 20 --causal 1 --S 1024 --h 25 --b 4 | tail -1
for c in 0 1; do timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:attn_bwd_persistent -c 2 --csv python tools/attn_bench.py --reps 2 --causal $c 2>/dev/null | grep -E "attn" | awk -F'","' '{print "bwd causal='$c'", $(NF)}' | head -2; done
