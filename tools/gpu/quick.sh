mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -rf -k "c2b or feature or canonical" > gpurun_out/pytest_quick.log 2>&1; echo "rc=$?"; tail -3 gpurun_out/pytest_quick.log
timeout 600 python tools/profile_variants.py --time c1 c2a c2b short band01 uvar3 c4 csr_vector > gpurun_out/quick.json 2>/dev/null
python -c "import json; t=json.load(open('gpurun_out/quick.json')); [print(c, round(r['feature_ms'],3), {k: (round(v['GBps']), round(v['ms'],4), v['tail']) for k,v in r['variants'].items()}) for c,r in t.items()]"
