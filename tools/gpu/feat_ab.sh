# feature-pass A/B: parity tests of the feature kernels + timings (features only) on the classes
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "feature or canonical or malformed" > gpurun_out/pytest_feat.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_feat.log
timeout 900 python tools/profile_variants.py --time c1 c2a c2b short band01 uvar3 band48 c4 none > gpurun_out/feat_ab.json 2>/dev/null
python -c "import json; t=json.load(open('gpurun_out/feat_ab.json')); [print(c, round(r['feature_ms'],4), round(r.get('feature_gpu_ms',0),4)) for c,r in t.items()]"
