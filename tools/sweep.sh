t() { timeout 300 python tools/profile_variants.py --time $1 $2 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: {k: round(v['GBps']) for k,v in r['variants'].items()} for c,r in t.items()})"; }
echo "HYB ls default"; t "c2b c0" hyb
echo "HYB ls W=8"; NITRO_HYB_W=8 t "c2b" hyb
echo "HYB old"; NITRO_HYB_LS=0 t "c2b" hyb
