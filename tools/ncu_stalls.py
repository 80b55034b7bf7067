"""Warp-state samples of one kernel from an ncu report (source page, SASS): the top instructions and
the samples / executions of every mbarrier wait, keyed by its shared-memory operand.

    python tools/ncu_stalls.py gpurun_out/ncu_gemm_qkv_fwd.ncu-rep > profiles/<name>.txt
"""
import collections
import csv
import io
import re
import subprocess
import sys


def main():
    raw = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    print(rows[0][1] if rows and len(rows[0]) > 1 else "")
    h, data = rows[1], rows[2:]
    ia, isrc = h.index("Address"), h.index("Source")
    iall, iex = h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
    val = lambda r, i: float(r[i] or 0) if len(r) > i else 0.0  # noqa: E731
    tot = sum(val(r, iall) for r in data)
    print(f"total warp samples {tot:.0f}")
    print("\n# top instructions by samples")
    for r in sorted(data, key=lambda r: -val(r, iall))[:15]:
        print(f"{val(r, iall):7.0f} {100 * val(r, iall) / tot:5.1f}%  {r[isrc][:90]}")
    addr = {r[ia]: k for k, r in enumerate(data)}
    smp, ex = collections.Counter(), collections.Counter()
    for k, r in enumerate(data):
        m = re.search(r"TRYWAIT P\d, \[(.*?)\]", r[isrc])
        if not m:
            continue
        s = val(r, iall)
        if k + 1 < len(data):
            nxt = data[k + 1]
            s += val(nxt, iall)
            mm = re.search(r"BRA (0x[0-9a-f]+)", nxt[isrc])
            if mm and mm.group(1) in addr:  # the retry loop the branch jumps to
                j = addr[mm.group(1)]
                s += sum(val(q, iall) for q in data[j:j + 3])
        smp[m.group(1)] += s
        ex[m.group(1)] += val(r, iex)
    print("\n# mbarrier waits: samples (incl. retry loop), try-wait executions, barrier operand")
    for key, v in smp.most_common(10):
        print(f"{v:7.0f} {ex[key]:10.0f}  {key}")


if __name__ == "__main__":
    main()
