# A/B of the x L2 persisting window (NITRO_L2_PERSIST) on the gather-heavy classes + ncu DRAM bytes
mkdir -p gpurun_out
for p in 0 1 0 1; do
  NITRO_L2_PERSIST=$p timeout 600 python tools/profile_variants.py --time c2b c2a uvar3 band01 > gpurun_out/ab_persist_$p.json 2>/dev/null
  echo "persist=$p"; python -c "import json; t=json.load(open('gpurun_out/ab_persist_$p.json')); [print(c, {k: round(v['GBps']) for k,v in r['variants'].items()}) for c,r in t.items()]"
done
for p in 0 1; do
  NITRO_L2_PERSIST=$p timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_sectors.sum \
    --clock-control none -k 'regex:k_(csr_vector|hyb_tail|ell|csr_scalar)' --csv --log-file gpurun_out/ncu_persist_$p.csv \
    python tools/profile_variants.py c2b c2a > /dev/null 2>&1
  echo "ncu persist=$p rc=$?"
  python - <<PY
import csv
rows = list(csv.reader(open('gpurun_out/ncu_persist_$p.csv')))
hdr = next(i for i, r in enumerate(rows) if r and r[0] == 'ID')
h = rows[hdr]
ki, mi, vi = h.index('Kernel Name'), h.index('Metric Name'), h.index('Metric Value')
cur = {}
for r in rows[hdr + 1:]:
    if len(r) <= vi: continue
    cur.setdefault((r[0], r[ki][:40]), {})[r[mi]] = r[vi]
for k, v in cur.items(): print(k, v)
PY
done
