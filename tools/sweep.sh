timeout 600 python -m pytest tests/test_gpu_hist.py -x -q 2>&1 | tail -2
python tools/hist_probe.py --time uniform; python tools/hist_probe.py --time spike; python tools/hist_probe.py --time normal
timeout 1500 python tools/hist_select.py --out gpurun_out/artifacts > gpurun_out/hist_select.log 2>&1; echo "hist rc=$?"
python -c "
import json; r=json.load(open('gpurun_out/artifacts/hist_report.json')); print({k:v for k,v in r.items() if k in ('nitro_pct_mean','share_ge_90','best_gbps_median','best_gbps_max','train_label_counts','always_variant_mean')})"
