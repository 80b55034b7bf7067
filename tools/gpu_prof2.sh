timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_m4.csv python tools/profile_step.py --layers 2 --steps 2 > /dev/null 2>&1
python tools/launch_shares.py gpurun_out/launches_m4.csv --last 500 | head -30
