# full gpu suite + smoke at HEAD
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r02_gpu_tests_final.txt 2>&1; echo "gpu tests $?"; tail -2 gpurun_out/r02_gpu_tests_final.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02_smoke_final.txt 2>&1; echo "smoke $?"; tail -1 gpurun_out/r02_smoke_final.txt
