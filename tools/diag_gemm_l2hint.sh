# output stores with an L2 evict_first policy (HARMONY_GEMM_DIAG=8) vs default, cfg2 shapes + K sweep
mkdir -p gpurun_out
timeout 300 python tools/gemm_bench.py --graph --reps 20 --cublas > gpurun_out/gb_r02_def.jsonl 2>&1
HARMONY_GEMM_DIAG=8 timeout 300 python tools/gemm_bench.py --graph --reps 20 > gpurun_out/gb_r02_ef.jsonl 2>&1
timeout 300 python tools/gemm_bench.py --sweep --graph --reps 20 > gpurun_out/sw_r02_def.jsonl 2>&1
HARMONY_GEMM_DIAG=8 timeout 300 python tools/gemm_bench.py --sweep --graph --reps 20 > gpurun_out/sw_r02_ef.jsonl 2>&1
python - <<'PY' | tee gpurun_out/r02_gemm_l2hint.txt
import json
def load(f):
    return {r["gemm"]: r for r in map(json.loads, (l for l in open(f) if l.startswith("{"))) if "us" in r}
for a_, b_ in (("gb_r02_def", "gb_r02_ef"), ("sw_r02_def", "sw_r02_ef")):
    a, b = load(f"gpurun_out/{a_}.jsonl"), load(f"gpurun_out/{b_}.jsonl")
    print("%-26s %9s %9s %9s" % ("shape", "default", "evict1st", "cuBLAS"))
    for k in a:
        print("%-26s %9.1f %9.1f %9.1f" % (k, a[k]["us"], b.get(k, {}).get("us", float("nan")), a[k].get("cublas_us", float("nan"))))
    print("total", sum(a[k]["us"] for k in a), sum(b[k]["us"] for k in b if k in a))
PY
