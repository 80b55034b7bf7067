# round 2, first GPU pass: the new group (N>1 loopback) tests, the >=4x-cap test, smoke, a short bench,
# the full gpu suite, compute-sanitizer logs.
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_group.py -m gpu -x -q -s > gpurun_out/t_group.log 2>&1; echo "group tests $?"; tail -3 gpurun_out/t_group.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -x -q -s -k over_4x > gpurun_out/t_4x.log 2>&1; echo "4x test $?"; tail -3 gpurun_out/t_4x.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke $?"; tail -2 gpurun_out/smoke.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench $?"; tail -c 600 gpurun_out/bench.json
for t in cfg1 tiny group; do
  HARMONY_NO_GRAPH=1 timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_step.py $t > gpurun_out/memcheck_$t.log 2>&1; echo "memcheck $t $?"; tail -3 gpurun_out/memcheck_$t.log
done
HARMONY_NO_GRAPH=1 timeout 900 compute-sanitizer --tool synccheck --print-limit 20 python tools/sanitize_step.py cfg1 group > gpurun_out/synccheck.log 2>&1; echo "synccheck $?"; tail -3 gpurun_out/synccheck.log
HARMONY_NO_GRAPH=1 timeout 1200 compute-sanitizer --tool racecheck --racecheck-report all --print-limit 20 python tools/sanitize_step.py cfg1 tiny > gpurun_out/racecheck.log 2>&1; echo "racecheck $?"; tail -3 gpurun_out/racecheck.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/t_all.log 2>&1; echo "all gpu tests $?"; tail -3 gpurun_out/t_all.log
