"""Summarise an ncu launch list (gpu__time_duration.sum per launch) into per-kernel shares.

    python tools/launch_shares.py gpurun_out/launches.csv [--last-step N]
"""
import csv
import re
import sys
from collections import defaultdict


def main():
    path = sys.argv[1]
    rows = []
    with open(path) as f:
        lines = [l for l in f if l.startswith('"')]
    for r in csv.DictReader(lines):
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(r["Metric Value"].replace(",", ""))
        unit = r.get("Metric Unit", "ns")
        scale = {"ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "nsecond": 1e-3}.get(unit, 1e-3)
        name = re.sub(r"\(.*", "", r["Kernel Name"]).replace("void ", "")
        name = re.sub(r"<.*", lambda m: m.group(0)[:40], name)
        rows.append((name, v * scale))
    if len(sys.argv) > 3 and sys.argv[2] == "--last":
        rows = rows[-int(sys.argv[3]):]
    tot = sum(t for _, t in rows)
    agg = defaultdict(lambda: [0, 0.0])
    for n, t in rows:
        agg[n][0] += 1
        agg[n][1] += t
    print(f"{len(rows)} launches, {tot:.1f} us total (serialised, cold-cache)")
    print(f"{'kernel':60s} {'launches':>8s} {'total us':>10s} {'avg us':>9s} {'share':>7s}")
    for n, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"{n[:60]:60s} {c:8d} {t:10.1f} {t / c:9.2f} {100 * t / tot:6.1f}%")


if __name__ == "__main__":
    main()
