mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 900 python -m pytest tests -m gpu -q -x -rf --durations=8 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/pytest_gpu.log
timeout 120 python __graft_entry__.py smoke 2>&1 | tail -1
timeout 300 ./tools/probes/l2_gather_probe > gpurun_out/l2_gather_probe.jsonl 2>&1; echo "probe rc=$?"; cat gpurun_out/l2_gather_probe.jsonl
timeout 600 python tools/profile_variants.py --time c1 c2a c2b short > gpurun_out/variant_table.json 2> gpurun_out/variant_table.err; echo "table rc=$?"
python -c "import json; t=json.load(open('gpurun_out/variant_table.json')); [print(c, round(r['feature_ms'],3), {k: round(v['GBps']) for k,v in r['variants'].items()}) for c,r in t.items()]"
