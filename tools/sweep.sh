t() { timeout 300 python tools/profile_variants.py --time $1 $2 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: {k: (round(v['GBps']), round(v['ms'],4)) for k,v in r['variants'].items()} for c,r in t.items()})"; }
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
M="c1 band48 band96h short band01 uvar3 c2a c2b"
for rep in 1 2; do
echo "STREAM=0"; NITRO_CSRV_STREAM=0 t "$M" "csr_vector"
for g in 4 8 16; do echo "STREAM=1 GRID=$g"; NITRO_CSRV_STREAM_GRID=$g t "$M" "csr_vector"; done
done
