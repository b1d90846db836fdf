mkdir -p gpurun_out
NITRO_CSRV_TMA=1 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -rf -k "stream or impls or misaligned or c2b" > gpurun_out/pytest_tma.log 2>&1; echo "rc=$?"; tail -3 gpurun_out/pytest_tma.log
for t in 0 1 0 1; do
  NITRO_CSRV_TMA=$t NITRO_CSRV_STREAM=1 timeout 600 python tools/profile_variants.py --time c2b c2a uvar3 csr_vector > gpurun_out/ab_tma.json 2>/dev/null
  echo "tma=$t"; python -c "import json; t=json.load(open('gpurun_out/ab_tma.json')); print(' '.join(f'{c}:{round(r[\"variants\"][\"csr_vector\"][\"ms\"],4)}' for c,r in t.items()))"
done
