# ncu metrics of the one- and two-query-tile attention forwards
mkdir -p gpurun_out
for k in 2 1; do
  HARMONY_ATTN_FWD=$k timeout 300 ncu --metrics gpu__time_duration.sum,sm__cycles_active.avg,smsp__inst_executed.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,smsp__inst_executed_pipe_xu.sum,gpc__cycles_elapsed.avg.per_second --clock-control none -k regex:attn_fwd -c 3 python tools/attn_bench.py --reps 2 --causal 0 --b 32 > gpurun_out/ncu_attn_fwd$k.txt 2>&1
  grep -E "attn_fwd|gpu__time|cycles_active|inst_executed|tensor|dram__|lts__t_bytes|per_second" gpurun_out/ncu_attn_fwd$k.txt | head -24
done
HARMONY_ATTN_FWD=2 timeout 600 ncu --set full --import-source on --clock-control none -k regex:attn_fwd2 -c 1 -s 2 -o gpurun_out/ncu_attn_fwd2_full -f python tools/attn_bench.py --reps 2 --causal 0 --b 32 > /dev/null 2>&1; echo "full $?"
