# timing of the persistent attention backward at 4 / 8 / 16 sub-tiles per item (1024 items)
for cfg in "--S 256 --b 32" "--S 512 --b 16" "--S 1024 --b 8"; do
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:attn_bwd_persistent -c 1 --csv python tools/attn_bench.py --reps 1 $cfg 2>/dev/null | grep -E "attn_bwd_persistent" | awk -F'","' '{print "'"$cfg"'", $(NF)}'
done
