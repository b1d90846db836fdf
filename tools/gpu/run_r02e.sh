mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -rf -k "impls or stream or misaligned" > gpurun_out/pytest_stream2.log 2>&1; echo "rc=$?"; tail -4 gpurun_out/pytest_stream2.log
for mode in 1; do
  NITRO_CSRV_STREAM=$mode timeout 600 python tools/profile_variants.py --time c2b c2a uvar3 band01 c1 short csr_vector > gpurun_out/stream2_$mode.json 2>/dev/null
  echo "stream=$mode"; python -c "import json; t=json.load(open('gpurun_out/stream2_$mode.json')); [print(c, {k: (round(v['GBps']), round(v['ms'],4)) for k,v in r['variants'].items()}) for c,r in t.items()]"
done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active --clock-control none -k 'regex:k_csr_stream' -c 2 --csv python tools/profile_variants.py c2b csr_vector 2>/dev/null | tail -8
