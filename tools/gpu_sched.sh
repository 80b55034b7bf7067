for w in cfg2 cfg3; do for sc in baseline harmony; do
timeout 900 python bench.py --workload $w --no-cpu-baseline --schedule $sc --steps 3 > gpurun_out/sched_${w}_$sc.json 2> gpurun_out/sched_${w}_$sc.err
python -c "import json;d=json.load(open('gpurun_out/sched_${w}_$sc.json'));sr=d['step_roofline'];print('$w $sc', round(d['value'],2), round(d['ms_per_step'],1), 'h2d', sr['h2d_bytes_per_step'], 'd2h', sr['d2h_bytes_per_step'], 'frac', round(sr['frac_strict'],3))" || tail -3 gpurun_out/sched_${w}_$sc.err
done; done
