# feature-pass timing (median of 7, L2 flushed) + full GPU suite
f() { timeout 300 python tools/profile_variants.py --time $1 none 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: round(r['feature_ms'],3) for c,r in t.items()})"; }
f "c0 c1 short c2a c2b"
timeout 1500 python -m pytest tests -q -x -m gpu 2>&1 | tail -3
