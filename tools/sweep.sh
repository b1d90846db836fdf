t() { timeout 300 python tools/profile_variants.py --time $1 $2 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: {k: round(v['GBps']) for k,v in r['variants'].items()} for c,r in t.items()}, {c: round(r['feature_ms'],3) for c,r in t.items()})"; }
echo "L2EF=1"; t "c1 c2a c2b" "ell hyb"
echo "L2EF=0"; NITRO_L2EF=0 t "c1 c2a c2b" "ell hyb"
