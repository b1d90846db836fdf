t() { timeout 300 python tools/profile_variants.py --time $1 $2 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: {k: (round(v['GBps']), round(v['ms'],4)) for k,v in r['variants'].items()} for c,r in t.items()})"; }
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
t "c1 c1big band48 c2a short" "ell hyb"
