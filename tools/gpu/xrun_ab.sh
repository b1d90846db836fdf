# K6v x-run vector loads: NITRO_K6V_XRUN=1 vs 0 (CSR-vector), interleaved; impl tests with it on
mkdir -p gpurun_out
NITRO_K6V_XRUN=1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "impls or misaligned or stencil or all_variants or c1 or c2a" > gpurun_out/pytest_xrun.log 2>&1; echo "pytest xrun rc=$?"; tail -2 gpurun_out/pytest_xrun.log
summ() { python -c "import json,sys; t=json.load(open(sys.argv[1])); print(' '.join(f'{c} '+' '.join(f'{v[\"GBps\"]:.0f}' for k,v in r['variants'].items()) for c,r in t.items()))" $1; }
CF=${CF:-c1 c1big band48 band96h short band01 uvar3 c2a c4}
for rep in 1 2; do
  timeout 900 python tools/profile_variants.py --time $CF csr_vector > gpurun_out/xr0.json 2>/dev/null; echo "xr0: $(summ gpurun_out/xr0.json)"
  NITRO_K6V_XRUN=1 timeout 900 python tools/profile_variants.py --time $CF csr_vector > gpurun_out/xr1.json 2>/dev/null; echo "xr1: $(summ gpurun_out/xr1.json)"
done
