t() { timeout 300 python tools/profile_variants.py --time $1 $2 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: {k: (round(v['GBps']), round(v['ms'],4)) for k,v in r['variants'].items()} for c,r in t.items()})"; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "csr or tolerance or integer or long_row or full" 2>&1 | tail -3
for rep in 1 2; do t "c1 band48 short band01 uvar3 c2a c2b" "csr_scalar csr_vector"; done
