mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -k "csr_impls or spmv_all or integer or long_row" > gpurun_out/pt13.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pt13.log
run() { env $1 timeout 600 python tools/profile_variants.py --time c1 short band01 uvar3 c2a c2b csr_vector > gpurun_out/v13.json 2>/dev/null
  echo "$1"; python -c "
import json; t=json.load(open('gpurun_out/v13.json'))
print({c: round(r['variants']['csr_vector']['GBps']) for c,r in t.items()})"; }
run NITRO_X=0
run NITRO_CSRV_DEEP=1
NITRO_CSRV_DEEP=1 timeout 900 python -m pytest tests -m gpu -q -x -k "csr_impls or spmv_all or integer or long_row" > gpurun_out/pt13b.log 2>&1; echo "pytest deep rc=$?"; tail -2 gpurun_out/pt13b.log
