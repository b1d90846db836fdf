# A/B of ab/libnitro_head.so vs the in-tree build (features on several classes,
# CSR-vector / HYB on c2b, fp64 EP 4 vs 8), interleaved, plus the GPU tests.
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -rf > gpurun_out/pytest_ab.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_ab.log
summ() { python - "$1" <<'PY'
import json,sys
t=json.load(open(sys.argv[1]))
print(' '.join(f'{c} F{r["feature_ms"]:.4f}/{(r.get("feature_gpu_ms") or 0):.4f} ' + ' '.join(f'{k}:{v["ms"]:.4f}' for k,v in r['variants'].items()) for c,r in t.items()))
PY
}
CF=${CFGS:-c1 c4 c2a c2b short band01 uvar3 band48}
for rep in 1 2; do
  NITRO_LIB=$PWD/ab/libnitro_head.so timeout 900 python tools/profile_variants.py --time $CF ${VARS:-none} > gpurun_out/ab_head.json 2>/dev/null
  echo "head: $(summ gpurun_out/ab_head.json)"
  timeout 900 python tools/profile_variants.py --time $CF ${VARS:-none} > gpurun_out/ab_new.json 2>/dev/null
  echo "new : $(summ gpurun_out/ab_new.json)"
done
for rep in 1 2; do
  NITRO_LIB=$PWD/ab/libnitro_head.so timeout 600 python tools/profile_variants.py --time c2b csr_vector hyb > gpurun_out/ab_head2.json 2>/dev/null
  echo "head c2b: $(summ gpurun_out/ab_head2.json)"
  timeout 600 python tools/profile_variants.py --time c2b csr_vector hyb > gpurun_out/ab_new2.json 2>/dev/null
  echo "new  c2b: $(summ gpurun_out/ab_new2.json)"
  NITRO_CSRV_EP64=8 timeout 600 python tools/profile_variants.py --time c2b csr_vector > gpurun_out/ab_ep8.json 2>/dev/null
  echo "ep8  c2b: $(summ gpurun_out/ab_ep8.json)"
done
