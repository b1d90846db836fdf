# tuning sweeps on c1 / c2a / c2b: ELL batch width, CSR-vector lane shift
t() { timeout 300 python tools/profile_variants.py --time $1 $2 2>/dev/null | python -c "import json,sys; t=json.load(sys.stdin); print({c: {k: round(v['GBps']) for k,v in r['variants'].items()} for c,r in t.items()})"; }
for u in 2 4 8; do echo "ELL U=$u"; NITRO_ELL_U=$u t "c1 c2a" ell; done
for sh in 0 1 2; do echo "CSRV shift=$sh"; NITRO_CSRV_SHIFT=$sh t "c1 c2a c2b" csr_vector; done
echo "DIA TMA"; NITRO_DIA_TMA=1 t "c1 short" dia; echo "DIA LDG"; t "c1 short" dia
