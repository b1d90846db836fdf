mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -rf -k "stream or impls or misaligned or c2b or long_row or spmv_all" > gpurun_out/pytest_hot.log 2>&1; echo "rc=$?"; tail -3 gpurun_out/pytest_hot.log
for h in 0 1 0 1; do
  NITRO_CSRV_HOT=$h timeout 600 python tools/profile_variants.py --time c2b csr_vector > gpurun_out/ab_hot.json 2>/dev/null
  echo "hot=$h"; python -c "import json; t=json.load(open('gpurun_out/ab_hot.json')); print(' '.join(f'{c}:{round(r[\"variants\"][\"csr_vector\"][\"ms\"],4)}/{round(r[\"variants\"][\"csr_vector\"][\"GBps\"])}' for c,r in t.items()))"
done
python - <<'PY'
import torch, synth, paper_conf_ipps_muralidharanshgc14_b200 as n
A = synth.rmat(23, 16, seed=7, fp64=True, device="cuda")
M = n.SpMV.from_csr(A); M.features(); M.prepare(n.CSR_VECTOR)
print("format", M.format_info(n.CSR_VECTOR))
PY
