mkdir -p gpurun_out
NITRO_FEAT_STREAM=1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -rf -k "feature or canonical or malformed" > gpurun_out/pytest_featstream.log 2>&1; echo "rc=$?"; tail -3 gpurun_out/pytest_featstream.log
for f in "NITRO_FEAT_STREAM=0" "NITRO_FEAT_STREAM=1 NITRO_FEAT_EP=8" "NITRO_FEAT_STREAM=1 NITRO_FEAT_EP=16"; do
  env $f timeout 600 python tools/profile_variants.py --time c1 c2a c2b uvar3 band01 short band48 c4 none > gpurun_out/featstream.json 2>/dev/null
  echo "$f"; python -c "import json; t=json.load(open('gpurun_out/featstream.json')); print(' '.join(f'{c}:{round(r[\"feature_ms\"],3)}' for c,r in t.items()))"
done
