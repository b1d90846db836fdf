# tuning sweeps: ELL batch width (c1, c2a), DIA batch width with vectorised x loads
t() { timeout 300 python tools/profile_variants.py --time $1 $2 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: {k: round(v['GBps']) for k,v in r['variants'].items()} for c,r in t.items()}, {c: round(r['feature_ms'],3) for c,r in t.items()})"; }
for u in 1 2; do echo "ELL U=$u"; NITRO_ELL_U=$u t "c1 c2a" ell; done
for u in 1 2 4 8; do echo "DIA U=$u"; NITRO_DIA_U=$u t "c1 short" dia; done
echo "all"; t "c1 c2a c2b short" ""
