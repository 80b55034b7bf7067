# is the forward bound by the strided Q/K/V tile reads of the packed [T, 3d] layout? same work, h = 16 vs h = 1
for k in 2 1; do
HARMONY_ATTN_FWD=$k timeout 120 python tools/attn_bench.py --reps 20 --causal 0 --b 32 --h 16 2>&1 | grep attn_fwd | sed "s/^/fwd$k h16 b32 /"
HARMONY_ATTN_FWD=$k timeout 120 python tools/attn_bench.py --reps 20 --causal 0 --b 512 --h 1 2>&1 | grep attn_fwd | sed "s/^/fwd$k h1 b512 /"
HARMONY_ATTN_FWD=$k timeout 120 python tools/attn_bench.py --reps 20 --causal 0 --b 128 --h 4 2>&1 | grep attn_fwd | sed "s/^/fwd$k h4 b128 /"
done
