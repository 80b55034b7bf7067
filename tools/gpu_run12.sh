set -x
timeout 600 python -m pytest tests/test_gpu_step.py -x -q 2>&1 | tail -3
timeout 900 python tools/timeline.py --workload cfg3 --out gpurun_out/timeline_cfg3.json > gpurun_out/timeline_cfg3.txt 2>&1
timeout 600 python tools/timeline.py --workload cfg2 --out gpurun_out/timeline_cfg2.json > gpurun_out/timeline_cfg2.txt 2>&1
for i in 1 2; do
  HARMONY_PRIO=0 timeout 600 python bench.py --no-cpu-baseline > gpurun_out/prio0_$i.json 2>/dev/null
  timeout 600 python bench.py --no-cpu-baseline > gpurun_out/prio1_$i.json 2>/dev/null
done
for f in gpurun_out/prio*.json; do python -c "import json;d=json.load(open('$f'));print('$f', round(d['value'],1))"; done
head -60 gpurun_out/timeline_cfg3.txt
