timeout 900 python -m pytest tests/test_gpu_hist.py -x -q 2>&1 | tail -3
timeout 1500 python tools/hist_select.py --out gpurun_out/artifacts > gpurun_out/hist_select.log 2>&1; echo "hist rc=$?"
