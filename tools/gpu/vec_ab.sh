# K6v (vector-load CSR-vector) A/B: AUTO with NITRO_CSRV_VEC=1 vs K6 (default), interleaved; impl tests first
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "impls or misaligned or c1 or c2a or c2b or stencil or long_row or all_variants" > gpurun_out/pytest_vec.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_vec.log
summ() { python -c "import json,sys; t=json.load(open(sys.argv[1])); print(' '.join(f'{c} '+' '.join(f'{k}:{v[\"ms\"]:.4f}/{v[\"GBps\"]:.0f}' for k,v in r['variants'].items()) for c,r in t.items()))" $1; }
CF=${CF:-c1 c1big band48 band96h short band01 uvar3 c2a c4}
for rep in 1 2; do
  timeout 900 python tools/profile_variants.py --time $CF csr_vector > gpurun_out/vec_k6.json 2>/dev/null; echo "k6 : $(summ gpurun_out/vec_k6.json)"
  NITRO_CSRV_VEC=1 timeout 900 python tools/profile_variants.py --time $CF csr_vector > gpurun_out/vec_k6v.json 2>/dev/null; echo "k6v: $(summ gpurun_out/vec_k6v.json)"
done
