# round-2 measurement suite at HEAD (one B200): traffic launch list + ncu full of the top GEMM, then every
# bench workload, the tuner and the reference arm
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r02_traffic_launches.csv python tools/profile_step.py --layers 2 --steps 2 > gpurun_out/ncu_traffic.log 2>&1; echo "ncu traffic $?"
python tools/traffic_summary.py gpurun_out/r02_traffic_launches.csv --last 158 > gpurun_out/r02_traffic_cfg2_m2.json; echo "traffic summary $?"
python tools/launch_shares.py gpurun_out/r02_traffic_launches.csv --last 158 > gpurun_out/r02_launch_shares_cfg2_m2.txt 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:gemm_tc2 -c 1 -s 3 -o gpurun_out/r02_ncu_full_gemm_qkv -f python tools/gemm_bench.py --only qkv_fwd --reps 3 > /dev/null 2>&1; echo "ncu full $?"
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r02_final_cfg2.json 2> gpurun_out/r02_final_cfg2.err; echo "cfg2 $?"
timeout 900 python bench.py --workload cfg3 --no-cpu-baseline --steps 5 > gpurun_out/r02_final_cfg3.json 2> gpurun_out/r02_final_cfg3.err; echo "cfg3 $?"
timeout 1500 python bench.py --workload cfg3s --no-cpu-baseline --steps 3 > gpurun_out/r02_final_cfg3s.json 2> gpurun_out/r02_final_cfg3s.err; echo "cfg3s $?"
timeout 1200 python bench.py --workload cfg4s --no-cpu-baseline --steps 3 > gpurun_out/r02_final_cfg4s.json 2> gpurun_out/r02_final_cfg4s.err; echo "cfg4s $?"
timeout 600 python bench.py --workload cfg1 --no-cpu-baseline > gpurun_out/r02_final_cfg1.json 2> gpurun_out/r02_final_cfg1.err; echo "cfg1 $?"
timeout 900 python bench.py --workload cfg5 --steps 3 > gpurun_out/r02_final_cfg5.json 2> gpurun_out/r02_final_cfg5.err; echo "cfg5 $?"
timeout 1500 python bench.py --tune --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r02_final_cfg2_tuned.json 2> gpurun_out/r02_final_cfg2_tuned.err; echo "tune $?"
SECONDS=0; timeout 1500 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/r02_final_ref.json 2> gpurun_out/r02_final_ref.err; echo "ref $? wall ${SECONDS}s"; tail -1 gpurun_out/r02_final_ref.err
for f in cfg2 cfg3 cfg3s cfg4s cfg1 cfg5 cfg2_tuned ref; do python -c "
import json
d=json.loads(open('gpurun_out/r02_final_$f.json').read().strip().splitlines()[-1])
sr=d.get('step_roofline') or {}
print('$f', d.get('value'), d.get('unit'), 'gemm_frac', (d.get('roofline') or {}).get('frac'), 'strict', sr.get('frac_strict'), 'cap_aware', (sr.get('cap_aware') or {}).get('frac'), 'e2e', (d.get('e2e') or {}).get('value'), (d.get('config') or {}).get('tuning', {}).get('best') if isinstance((d.get('config') or {}).get('tuning'), dict) else '')
"; done
