# Which epilogue resource slows the mainloop: the K sweep with HARMONY_GEMM_DIAG = 1 (epilogue drains
# nothing), 2 (no TMEM loads: zeros stored), 4 (TMEM loads, no TMA store of the output)
mkdir -p gpurun_out
timeout 300 python tools/gemm_bench.py --sweep --graph --reps 20 --cublas > gpurun_out/sweep_r02_default.jsonl 2>&1
for d in 1 2 4 6; do HARMONY_GEMM_DIAG=$d timeout 300 python tools/gemm_bench.py --sweep --graph --reps 20 > gpurun_out/sweep_r02_diag$d.jsonl 2>&1; done
python - <<'PY' | tee gpurun_out/sweep_r02_diag_summary.txt
import json
def load(f):
    return {r["gemm"]: r for r in map(json.loads, (l for l in open(f) if l.startswith("{"))) if "us" in r}
a = load("gpurun_out/sweep_r02_default.jsonl")
d = {k: load(f"gpurun_out/sweep_r02_diag{k}.jsonl") for k in (1, 2, 4, 6)}
print("%-26s %9s %9s %9s %9s %9s %9s" % ("shape", "default", "no-epi", "no-ldtm", "no-store", "neither", "cuBLAS"))
for k in a:
    print("%-26s %9.1f %9.1f %9.1f %9.1f %9.1f %9.1f" % (k, a[k]["us"], *[d[x].get(k, {}).get("us", float("nan")) for x in (1, 2, 4, 6)], a[k].get("cublas_us", float("nan"))))
PY
