# re-validate HEAD on a fresh box: full gpu suite, smoke, default bench, launch list of a 2-layer step
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/r02_gpu_tests_head_c.txt 2>&1; echo "tests exit $?"
tail -3 gpurun_out/r02_gpu_tests_head_c.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 900 python bench.py > gpurun_out/r02_bench_head_c.json 2> gpurun_out/r02_bench_head_c.err; echo "bench exit $?"
tail -c 600 gpurun_out/r02_bench_head_c.json
