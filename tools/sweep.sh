# tuning sweeps: DIA split x batch, HYB tail windows
t() { timeout 300 python tools/profile_variants.py --time $1 $2 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: {k: round(v['GBps']) for k,v in r['variants'].items()} for c,r in t.items()})"; }
for ds in 1 2 4; do for u in 1 2; do echo "DIA DS=$ds U=$u"; NITRO_DIA_DS=$ds NITRO_DIA_U=$u t "c1 short" dia; done; done
for w in 2 4 8; do echo "HYB W=$w"; NITRO_HYB_W=$w t "c2b" hyb; done
