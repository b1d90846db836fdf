t() { timeout 300 python tools/profile_variants.py --time $1 $2 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: {k: (round(v['GBps']), round(v['ms'],4)) for k,v in r['variants'].items()} for c,r in t.items()})"; }
for rep in 1 2; do for pf in 0 1 2 4; do echo "HYB_PF=$pf"; NITRO_HYB_PF=$pf t "c2b uvar3 band01" "hyb"; done; done
NITRO_HYB_PF=2 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "tolerance or long_row or c2b or integer" 2>&1 | tail -2
