set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -30 > gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python tools/profile_step.py --layers 2 --steps 2 > gpurun_out/prof_step.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:'gemm_tc2|attn_fwd|attn_bwd|ln_fwd|ln_bwd|adam' -c 12 -o gpurun_out/full python tools/profile_step.py --layers 1 --steps 1 > gpurun_out/ncu_full.log 2>&1
tail -3 gpurun_out/pytest_gpu.log; cat gpurun_out/bench.json
