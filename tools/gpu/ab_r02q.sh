mkdir -p gpurun_out
NITRO_FEAT_MATCH=1 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "feature or canonical" > gpurun_out/pytest_match.log 2>&1; echo "rc=$?"; tail -2 gpurun_out/pytest_match.log
for m in 0 1 0 1; do
  NITRO_FEAT_MATCH=$m timeout 600 python tools/profile_variants.py --time c1 c2a short band01 uvar3 c4 none > gpurun_out/ab_match.json 2>/dev/null
  echo "match=$m"; python -c "import json; t=json.load(open('gpurun_out/ab_match.json')); print(' '.join(f'{c}:{round(r[\"feature_ms\"],3)}' for c,r in t.items()))"
done
