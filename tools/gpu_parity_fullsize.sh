mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_parity.py -q -s -k "full or step_parity_against" > gpurun_out/par.log 2>&1; echo "rc=$?"
tail -30 gpurun_out/par.log
