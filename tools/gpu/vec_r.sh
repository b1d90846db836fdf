# K6v rows-in-flight A/B: R = 2 (in-tree) vs ab/libnitro_r4.so / r8 (fp32), AUTO forced to K6v
mkdir -p gpurun_out
summ() { python -c "import json,sys; t=json.load(open(sys.argv[1])); print(' '.join(f'{c} '+' '.join(f'{v[\"GBps\"]:.0f}' for k,v in r['variants'].items()) for c,r in t.items()))" $1; }
CF=${CF:-c1 c1big band48 band96h short band01 uvar3 c2a c4}
for rep in 1 2; do
  NITRO_CSRV_VEC=1 timeout 900 python tools/profile_variants.py --time $CF csr_vector > gpurun_out/vr2.json 2>/dev/null; echo "r2: $(summ gpurun_out/vr2.json)"
  for L in r4 r8; do
    NITRO_LIB=$PWD/ab/libnitro_$L.so NITRO_CSRV_VEC=1 timeout 900 python tools/profile_variants.py --time $CF csr_vector > gpurun_out/v$L.json 2>/dev/null; echo "$L: $(summ gpurun_out/v$L.json)"
  done
done
