for e in 1 0; do
  echo "TMA_EPI=$e"
  HARMONY_GEMM_TMA_EPI=$e python tools/gemm_bench.py --graph 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print(d['gemm'], round(d.get('us',0),1), round(d['tflops']))"
done
