# DIA batch-width sweep (NITRO_DIA_U) on c1 and the short-row stencil
for u in 1 2 4 8; do
  echo "U=$u"; NITRO_DIA_U=$u timeout 300 python tools/profile_variants.py --time c1 short dia 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: round(r['variants']['dia']['GBps']) for c,r in t.items()})"
done
