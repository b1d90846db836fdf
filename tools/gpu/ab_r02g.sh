mkdir -p gpurun_out
NITRO_CSRV_STREAM=1 timeout 600 python tools/profile_variants.py --time c2b csr_vector > gpurun_out/stream_occ8.json 2>/dev/null
python -c "import json; t=json.load(open('gpurun_out/stream_occ8.json')); [print(c, {k: (round(v['GBps']), round(v['ms'],4)) for k,v in r['variants'].items()}) for c,r in t.items()]"
for t in 0 1; do
  NITRO_FEAT_TBS=$t timeout 600 python tools/profile_variants.py --time c2a c2b c1 uvar3 none > gpurun_out/feat_tbs_$t.json 2>/dev/null
  echo "tbs=$t"; python -c "import json; t=json.load(open('gpurun_out/feat_tbs_$t.json')); [print(c, round(r['feature_ms'],3)) for c,r in t.items()]"
done
