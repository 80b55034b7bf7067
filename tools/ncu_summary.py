"""Summarise an ncu report (raw page) into the metrics the roofline uses.

    python tools/ncu_summary.py gpurun_out/prof.ncu-rep [--grep REGEX] > profiles/<name>.txt
"""
import csv
import io
import re
import subprocess
import sys

KEYS = [
    "Kernel Name", "gpu__time_duration.sum", "launch__grid_size", "launch__block_size", "launch__registers_per_thread",
    "launch__shared_mem_per_block_dynamic", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
    "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
    "sm__mem_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "lts__t_bytes.sum", "l1tex__t_bytes.sum", "sm__cycles_elapsed.avg.per_second",
    "sm__ops_path_tensor_op_utchmma_src_bf16_dst_fp32_sparsity_off.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed", "sm__cycles_active.avg", "gpc__cycles_elapsed.max",
]


def main():
    path = sys.argv[1]
    pat = re.compile(sys.argv[3]) if len(sys.argv) > 3 and sys.argv[2] == "--grep" else None
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    if len(rows) < 3:
        print("no data", raw[:500])
        return
    head, units = rows[0], rows[1]
    for r in rows[2:]:
        print("-" * 80)
        for i, n in enumerate(head):
            if n in KEYS or (pat and pat.search(n)):
                print(f"{n:90s} {r[i]:>20s} {units[i]}")


if __name__ == "__main__":
    main()
