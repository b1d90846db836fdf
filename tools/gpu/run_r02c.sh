mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_itune.py tests/test_gpu_parity.py -q -x -rf --durations=5 > gpurun_out/pytest_itune.log 2>&1; echo "rc=$?"; tail -12 gpurun_out/pytest_itune.log
