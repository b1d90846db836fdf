mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x -rf --durations=8 > gpurun_out/pytest_full.log 2>&1; echo "rc=$?"; tail -16 gpurun_out/pytest_full.log
NITRO_CSRV_STREAM=1 timeout 600 python tools/profile_variants.py --time c2b c2a uvar3 band01 csr_vector > gpurun_out/stream3.json 2>/dev/null
python -c "import json; t=json.load(open('gpurun_out/stream3.json')); [print(c, {k: (round(v['GBps']), round(v['ms'],4)) for k,v in r['variants'].items()}) for c,r in t.items()]"
