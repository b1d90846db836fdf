mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -rf --durations=6 > gpurun_out/pytest_full.log 2>&1; echo "rc=$?"; tail -12 gpurun_out/pytest_full.log
timeout 120 python __graft_entry__.py smoke 2>&1 | tail -1
