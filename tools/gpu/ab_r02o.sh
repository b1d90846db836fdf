for t in 0 1; do
  NITRO_CSRV_STREAM=$t timeout 600 python tools/profile_variants.py --time band48 band96h c1big c1 csr_vector > gpurun_out/ab_long.json 2>/dev/null
  echo "stream=$t"; python -c "import json; t=json.load(open('gpurun_out/ab_long.json')); print(' '.join(f'{c}:{round(r[\"variants\"][\"csr_vector\"][\"ms\"],4)}/{round(r[\"variants\"][\"csr_vector\"][\"GBps\"])}' for c,r in t.items()))"
done
