# A/B of the feature pass: ab/libnitro_<name>.so vs the in-tree build, interleaved, same box
mkdir -p gpurun_out
CF=${CFGS:-c1 c2a c2b short band01 uvar3 band48 c4}
for rep in 1 2; do
  for lib in ${LIBS:-head}; do
    NITRO_LIB=$PWD/ab/libnitro_$lib.so timeout 900 python tools/profile_variants.py --time $CF none > gpurun_out/ab_$lib.json 2>/dev/null
    echo "$lib: $(python -c "import json; t=json.load(open('gpurun_out/ab_$lib.json')); print(' '.join(f'{c} {r[\"feature_ms\"]:.4f}/{r.get(\"feature_gpu_ms\",0):.4f}' for c,r in t.items()))")"
  done
  timeout 900 python tools/profile_variants.py --time $CF none > gpurun_out/ab_new.json 2>/dev/null
  echo "new: $(python -c "import json; t=json.load(open('gpurun_out/ab_new.json')); print(' '.join(f'{c} {r[\"feature_ms\"]:.4f}/{r.get(\"feature_gpu_ms\",0):.4f}' for c,r in t.items()))")"
done
