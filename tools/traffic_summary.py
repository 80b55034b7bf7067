"""Per-kernel-class DRAM traffic and time from an ncu launch list of the bench step.

    ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
        --csv --log-file gpurun_out/traffic.csv python tools/profile_step.py --layers 2 --steps 2
    python tools/traffic_summary.py gpurun_out/traffic.csv --last 850 > profiles/<round>_traffic_cfg2.json

ncu replays every kernel with its caches flushed (cold), so `dram_bytes_per_launch` is the traffic a
launch moves from HBM when nothing it reads is L2-resident — the upper end of what the step sees.
The "gemm" class matches the bench's roofline kernel class (the tcgen05 GEMMs of the step); the
fused attention kernels are their own class, as in the bench's profile.
"""
import csv
import json
import re
import sys
from collections import defaultdict

CLASSES = [("gemm", re.compile(r"gemm_tc")),
           ("attention", re.compile(r"attn_fwd|attn_bwd_persistent|attn_bwd_kernel")),
           ("layernorm", re.compile(r"ln_fwd|ln_bwd|colreduce2")),
           ("adam", re.compile(r"adam")),
           ("other", re.compile(r"."))]


def main():
    path = sys.argv[1]
    last = int(sys.argv[sys.argv.index("--last") + 1]) if "--last" in sys.argv else None
    with open(path) as f:
        lines = [l for l in f if l.startswith('"')]
    launches = defaultdict(dict)
    order = []
    for r in csv.DictReader(lines):
        key = (r["ID"], r["Kernel Name"])
        if key not in launches:
            order.append(key)
        v = float(r["Metric Value"].replace(",", ""))
        u = r.get("Metric Unit", "")
        scale = {"ns": 1e-9, "nsecond": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3, "msecond": 1e-3,
                 "byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}.get(u, 1)
        launches[key][r["Metric Name"]] = v * scale
    if last:
        order = order[-last:]
    agg = defaultdict(lambda: {"launches": 0, "seconds": 0.0, "dram_bytes": 0.0})
    per_kernel = defaultdict(lambda: {"launches": 0, "seconds": 0.0, "dram_bytes": 0.0})
    for key in order:
        m = launches[key]
        name = re.sub(r"\(.*", "", key[1]).replace("void ", "")
        cls = next(c for c, rx in CLASSES if rx.search(name))
        b = m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
        for d in (agg[cls], per_kernel[name]):
            d["launches"] += 1
            d["seconds"] += m.get("gpu__time_duration.sum", 0.0)
            d["dram_bytes"] += b
    tot = sum(d["seconds"] for d in agg.values())
    out = {"source": path, "launches": len(order), "serialised_seconds": tot, "classes": {}, "kernels": {}}
    for name, d in list(agg.items()) + list(per_kernel.items()):
        tgt = out["classes"] if name in agg and name in dict(CLASSES) else out["kernels"]
        tgt[name] = dict(d, dram_bytes_per_launch=d["dram_bytes"] / d["launches"], share=d["seconds"] / tot,
                         achieved_dram_gbs=d["dram_bytes"] / d["seconds"] / 1e9 if d["seconds"] else None)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
