t() { timeout 300 python tools/profile_variants.py --time $1 $2 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: {k: (round(v['GBps']), round(v['ms'],3)) for k,v in r['variants'].items()} for c,r in t.items()})"; }
for w in 4 8; do echo "HYB_W=$w"; NITRO_HYB_W=$w t "c2b" "hyb"; done
