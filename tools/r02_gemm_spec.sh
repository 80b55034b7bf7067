# A/B: per-epilogue-kind GEMM kernels vs the generic one (HARMONY_GEMM_SPECIALIZE=0); kernel tests; cfg2 bench
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
for sp in 1 0; do
HARMONY_GEMM_SPECIALIZE=$sp timeout 300 python tools/gemm_bench.py --reps 20 > gpurun_out/r02_gemm_spec$sp.jsonl 2>&1; echo "bench $sp $?"
done
python - <<'PY'
import json
def rd(f):
    d={}
    for l in open(f):
        try: j=json.loads(l)
        except Exception: continue
        d[j['gemm']]=j
    return d
a=rd('gpurun_out/r02_gemm_spec1.jsonl'); b=rd('gpurun_out/r02_gemm_spec0.jsonl')
ta=tb=0
for k in a:
    if k=='ALL': continue
    ta+=a[k]['us']; tb+=b[k]['us']
    print(f"{k:20s} spec {a[k]['us']:7.1f}  generic {b[k]['us']:7.1f}")
print('total', round(ta,1), round(tb,1))
PY
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_step.py -q -x -p no:cacheprovider 2>&1 | tail -3
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/r02_bench_spec.json 2> gpurun_out/r02_bench_spec.err; echo "bench cfg2 $?"
python -c "
import json
d=json.loads(open('gpurun_out/r02_bench_spec.json').read().strip().splitlines()[-1])
print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['step_roofline']['frac_strict'], d['clocks'])"
