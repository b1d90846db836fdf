t() { timeout 300 python tools/profile_variants.py --time $1 $2 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: {k: (round(v['GBps']), round(v['ms'],4)) for k,v in r['variants'].items()} for c,r in t.items()})"; }
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -1
t "c1 c1big band48" "ell hyb"
timeout 1200 python tools/c4_probe.py --out gpurun_out/c4_probe.json > gpurun_out/c4_probe.log 2>&1; echo "c4 rc=$?"; grep "^ell\|^dia\|^hyb" gpurun_out/c4_probe.log
