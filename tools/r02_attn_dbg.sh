# attention forward debug runs (single item, small grids)
mkdir -p gpurun_out
HARMONY_ATTN_GRID=1 timeout 60 python tools/attn_bench.py --reps 1 --causal 0 --b 1 --h 1 --S 512 2>&1 | grep -v "^  |Search|CUDA kernel|For debug|Compile with" | head -12
HARMONY_ATTN_GRID=1 timeout 60 python tools/attn_bench.py --reps 1 --causal 0 --b 1 --h 2 --S 256 2>&1 | grep -v "^  |Search|CUDA kernel|For debug|Compile with" | head -12
timeout 60 python tools/attn_bench.py --reps 1 --causal 0 --b 32 --h 16 --S 512 2>&1 | grep -v "^  |Search|CUDA kernel|For debug|Compile with" | head -12
