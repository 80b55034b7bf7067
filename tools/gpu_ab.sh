# A/B of two in-tree builds in one job: bench (alternating) + GEMM shapes under graph replay
set -x
A=abl/libharmony_f8867c2.so
for i in 1 2; do
  HARMONY_LIB=$A timeout 600 python bench.py --no-cpu-baseline > gpurun_out/ab_base_$i.json 2>/dev/null
  timeout 600 python bench.py --no-cpu-baseline > gpurun_out/ab_new_$i.json 2>/dev/null
done
HARMONY_LIB=$A timeout 300 python tools/gemm_bench.py --graph > gpurun_out/ab_gb_base.log 2>&1
timeout 300 python tools/gemm_bench.py --graph > gpurun_out/ab_gb_new.log 2>&1
for f in gpurun_out/ab_*.json; do python -c "import json;d=json.load(open('$f'));print('$f', round(d['value'],1), {k: round(v['per_launch_us'] or 0,2) for k,v in d['kernels'].items()})"; done
for f in ab_gb_base ab_gb_new; do echo "== $f"; grep -v Warn gpurun_out/$f.log | python -c "
import sys,json
out=[]
for l in sys.stdin:
    try: d=json.loads(l)
    except: continue
    out.append(f\"{d['gemm']}:{d.get('us',0):.1f}\")
print(' '.join(out))
"; done
