mkdir -p gpurun_out
NITRO_FEAT_STREAM=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_c4.py tests/test_gpu_dist_loopback.py -q -x -rf -k "feature or canonical or c1 or c2 or c4 or loopback_ranks or malformed" > gpurun_out/pytest_featstream.log 2>&1; echo "rc=$?"; tail -6 gpurun_out/pytest_featstream.log
for f in 0 1; do
  NITRO_FEAT_STREAM=$f timeout 600 python tools/profile_variants.py --time c1 c2a c2b uvar3 band01 short band48 c4 none > gpurun_out/featstream_$f.json 2>/dev/null
  echo "feat_stream=$f"; python -c "import json; t=json.load(open('gpurun_out/featstream_$f.json')); [print(c, round(r['feature_ms'],3), round(r['feature_GBps'])) for c,r in t.items()]"
done
