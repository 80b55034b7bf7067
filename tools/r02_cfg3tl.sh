# op timeline of a cfg3 step
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 900 python tools/timeline.py --workload cfg3 > gpurun_out/r02_timeline_cfg3.json 2>&1; echo "tl $?"
