# Harmony-PP, step and group test suites
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_pp.py -m gpu -x -q -s > gpurun_out/t_pp.log 2>&1; echo "pp tests $?"; tail -6 gpurun_out/t_pp.log
timeout 1200 python -m pytest tests/test_gpu_step.py tests/test_gpu_group.py -m gpu -x -q > gpurun_out/t_step.log 2>&1; echo "step+group tests $?"; tail -3 gpurun_out/t_step.log
HARMONY_NO_GRAPH=1 timeout 600 compute-sanitizer --tool memcheck --print-limit 20 python -c "
import sys; sys.path.insert(0, '.')
import synth
from paper_conf_hotos_lipmk21_b200 import harmony as H
descs = synth.transformer_stack(4, 128, 2, 128, True)
params = synth.gen_params(descs, 1)
X, T = synth.gen_batch(descs, 4, 1, 1)
with H.Harmony(descs, params, group=[0, 0], schedule=H.HARMONY_SCHED_HARMONY_PP, microbatches=2, microbatch_size=2, precision=1, stash_policy=2) as h:
    print('pp loss', h.step(X, T)[0])
" > gpurun_out/memcheck_pp.log 2>&1; echo "memcheck pp $?"; tail -2 gpurun_out/memcheck_pp.log
