# attention kernel time vs item count (one item per CTA and multiples), S=512, 4 key / 4 query tiles per (b, h)
for cfg in "--S 512 --b 37 --h 1" "--S 512 --b 74 --h 1" "--S 512 --b 148 --h 1" "--S 512 --b 16 --h 16"; do
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:attn_ -c 3 --csv python tools/attn_bench.py --reps 1 $cfg 2>/dev/null | grep -E "attn_fwd_kernel|attn_bwd_persistent" | sed -E 's/.*(attn_fwd_kernel|attn_bwd_persistent).*,"([0-9.]+)"$/\1 \2/' | sed "s/^/$cfg /"
done
