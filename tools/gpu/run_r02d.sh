mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_itune.py tests/test_gpu_parity.py -q -x -rf --durations=5 -k "itune or timeout or impls or stream or misaligned or spmv_all or long_row or c2b" > gpurun_out/pytest_stream.log 2>&1; echo "rc=$?"; tail -12 gpurun_out/pytest_stream.log
for mode in 0 1; do
  NITRO_CSRV_STREAM=$mode timeout 600 python tools/profile_variants.py --time c2b c2a uvar3 band01 c1 short csr_vector > gpurun_out/stream_$mode.json 2>/dev/null
  echo "stream=$mode"; python -c "import json; t=json.load(open('gpurun_out/stream_$mode.json')); [print(c, {k: (round(v['GBps']), round(v['ms'],4)) for k,v in r['variants'].items()}) for c,r in t.items()]"
done
