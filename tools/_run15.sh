mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -k "feature or canonical or c4_features" > gpurun_out/pt15.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pt15.log
timeout 600 python tools/profile_variants.py --time c1 short band01 uvar3 c2a c2b none > gpurun_out/f15.json 2>/dev/null
python -c "
import json; t=json.load(open('gpurun_out/f15.json'))
print({c: (round(r['feature_ms'],3), round(r['feature_GBps'])) for c,r in t.items()})"
