# Per-tile epilogue exposure of the CTA-pair GEMM: K sweep (256..4096) of the QKV / FC1 shapes with a
# bf16 store, an fp32 store and the two-output BIAS_ACT epilogue, for the default 256x256 pair tiles,
# 256x128 pair tiles (HARMONY_GEMM_2SM=3) and the register epilogue (HARMONY_GEMM_TMA_EPI=0); cuBLAS beside.
#   gpurun --timeout 900 -- 'bash tools/diag_gemm_epi.sh'
mkdir -p gpurun_out
timeout 300 python tools/gemm_bench.py --sweep --graph --reps 20 --cublas > gpurun_out/sweep_default.jsonl 2>&1
HARMONY_GEMM_2SM=3 timeout 300 python tools/gemm_bench.py --sweep --graph --reps 20 > gpurun_out/sweep_2sm3.jsonl 2>&1
HARMONY_GEMM_TMA_EPI=0 timeout 300 python tools/gemm_bench.py --sweep --graph --reps 20 > gpurun_out/sweep_regepi.jsonl 2>&1
python - <<'PY' | tee gpurun_out/sweep_summary.txt
import json
def load(f):
    return {r["gemm"]: r for r in map(json.loads, (l for l in open(f) if l.startswith("{"))) if "us" in r}
d, t, g = load("gpurun_out/sweep_default.jsonl"), load("gpurun_out/sweep_2sm3.jsonl"), load("gpurun_out/sweep_regepi.jsonl")
print("%-24s %9s %9s %9s %9s   (us; TFLOP/s default)" % ("shape", "256x256", "256x128", "reg-epi", "cuBLAS"))
for k, r in d.items():
    print("%-24s %9.1f %9.1f %9.1f %9s   %.0f" % (k, r["us"], t.get(k, {}).get("us", float("nan")), g.get(k, {}).get("us", float("nan")),
          "%.1f" % r["cublas_us"] if "cublas_us" in r else "-", r["tflops"]))
PY
