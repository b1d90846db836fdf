mkdir -p gpurun_out
for cfg in "NITRO_CSRV_EP=4 NITRO_HYB_W=4" "NITRO_CSRV_EP=8 NITRO_HYB_W=8" "NITRO_CSRV_EP=4 NITRO_HYB_W=4" "NITRO_CSRV_EP=8 NITRO_HYB_W=8"; do
  env $cfg timeout 600 python tools/profile_variants.py --time c2b csr_vector hyb > gpurun_out/ab_ep.json 2>/dev/null
  echo "$cfg"; python -c "import json; t=json.load(open('gpurun_out/ab_ep.json')); [print(c, {k: (round(v['GBps']), round(v['ms'],4)) for k,v in r['variants'].items()}) for c,r in t.items()]"
done
for cfg in "NITRO_CSRV_EP=8" "NITRO_CSRV_EP=4"; do
  env NITRO_CSRV_STREAM=1 $cfg timeout 600 python tools/profile_variants.py --time c2a uvar3 csr_vector > gpurun_out/ab_ep2.json 2>/dev/null
  echo "$cfg fp32"; python -c "import json; t=json.load(open('gpurun_out/ab_ep2.json')); [print(c, {k: (round(v['GBps']), round(v['ms'],4)) for k,v in r['variants'].items()}) for c,r in t.items()]"
done
