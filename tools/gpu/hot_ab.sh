# A/B of the hot-x set size of K6s on configs[2] R-MAT (c2b)
for rep in 1 2; do
for kb in ${KBS:-64 80 96}; do
  echo "kb=$kb $(NITRO_CSRV_HOT_KB=$kb timeout 600 python tools/profile_variants.py --time c2b csr_vector 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print(round(t['c2b']['variants']['csr_vector']['ms'],4))")"
done; done
