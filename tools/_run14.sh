mkdir -p gpurun_out
run() { env $1 timeout 600 python tools/profile_variants.py --time c1 short band01 uvar3 c2a c2b csr_vector > gpurun_out/v14.json 2>/dev/null
  echo "$1"; python -c "
import json; t=json.load(open('gpurun_out/v14.json'))
print({c: round(r['variants']['csr_vector']['GBps']) for c,r in t.items()})"; }
run NITRO_X=0
run NITRO_CSRV_MINB=5
run NITRO_CSRV_MINB=6
