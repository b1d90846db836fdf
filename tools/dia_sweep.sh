# DIA implementation sweep: LDG kernel (NITRO_DIA_U batch widths) vs TMA-streamed kernel
for u in 2 4; do
  echo "LDG U=$u"; NITRO_DIA_U=$u timeout 300 python tools/profile_variants.py --time c1 short dia 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: round(r['variants']['dia']['GBps']) for c,r in t.items()})"
done
echo "TMA"; NITRO_DIA_TMA=1 timeout 300 python tools/profile_variants.py --time c1 short dia 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: round(r['variants']['dia']['GBps']) for c,r in t.items()})"
