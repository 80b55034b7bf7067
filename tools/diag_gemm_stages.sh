# 4 vs 5 mainloop stages of the CTA-pair GEMM (the bias no longer staged in shared memory), K sweep + cfg2 shapes
mkdir -p gpurun_out
timeout 300 python tools/gemm_bench.py --sweep --graph --reps 20 --cublas > gpurun_out/sweep_r02_s4.jsonl 2>&1
HARMONY_GEMM_STAGES=5 timeout 300 python tools/gemm_bench.py --sweep --graph --reps 20 > gpurun_out/sweep_r02_s5.jsonl 2>&1
timeout 300 python tools/gemm_bench.py --graph --reps 20 --cublas > gpurun_out/gb_r02_s4.jsonl 2>&1
HARMONY_GEMM_STAGES=5 timeout 300 python tools/gemm_bench.py --graph --reps 20 > gpurun_out/gb_r02_s5.jsonl 2>&1
python - <<'PY' | tee gpurun_out/sweep_r02_stages_summary.txt
import json
def load(f):
    return {r["gemm"]: r for r in map(json.loads, (l for l in open(f) if l.startswith("{"))) if "us" in r}
for a_, b_ in (("sweep_r02_s4", "sweep_r02_s5"), ("gb_r02_s4", "gb_r02_s5")):
    a, b = load(f"gpurun_out/{a_}.jsonl"), load(f"gpurun_out/{b_}.jsonl")
    print("%-26s %9s %9s %9s" % ("shape", "4 stages", "5 stages", "cuBLAS"))
    for k in a:
        print("%-26s %9.1f %9.1f %9.1f" % (k, a[k]["us"], b.get(k, {}).get("us", float("nan")), a[k].get("cublas_us", float("nan"))))
    print("total", sum(a[k]["us"] for k in a), sum(b[k]["us"] for k in b if k in a))
PY
timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q 2>&1 | tail -2
HARMONY_GEMM_STAGES=5 timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q 2>&1 | tail -2
