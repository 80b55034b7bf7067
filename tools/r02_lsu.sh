# GEMM epilogue through LSU stores vs TMA stores (HARMONY_GEMM_DIAG=16)
timeout 300 python tools/gemm_bench.py --graph --reps 20 > gpurun_out/gb_r02_tma.jsonl 2>&1
HARMONY_GEMM_DIAG=16 timeout 300 python tools/gemm_bench.py --graph --reps 20 > gpurun_out/gb_r02_lsu.jsonl 2>&1
timeout 300 python tools/gemm_bench.py --sweep --graph --reps 20 > gpurun_out/sw_r02_tma.jsonl 2>&1
HARMONY_GEMM_DIAG=16 timeout 300 python tools/gemm_bench.py --sweep --graph --reps 20 > gpurun_out/sw_r02_lsu.jsonl 2>&1
python - <<'PY' | tee gpurun_out/r02_gemm_lsu_stores.txt
import json
def load(f):
    return {r["gemm"]: r for r in map(json.loads, (l for l in open(f) if l.startswith("{"))) if "us" in r}
for a_, b_ in (("gb_r02_tma", "gb_r02_lsu"), ("sw_r02_tma", "sw_r02_lsu")):
    a, b = load(f"gpurun_out/{a_}.jsonl"), load(f"gpurun_out/{b_}.jsonl")
    print("%-26s %9s %9s" % ("shape", "TMA store", "LSU store"))
    for k in a:
        print("%-26s %9.1f %9.1f" % (k, a[k]["us"], b.get(k, {}).get("us", float("nan"))))
    print("total", round(sum(a[k]["us"] for k in a), 1), round(sum(b[k]["us"] for k in b if k in a), 1))
PY
HARMONY_GEMM_DIAG=16 timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q 2>&1 | tail -1
