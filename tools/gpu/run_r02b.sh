mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv,noheader
timeout 900 python -m pytest tests/test_gpu_dist_loopback.py tests/test_gpu_dist.py -q -x -rf --durations=5 > gpurun_out/pytest_loopback.log 2>&1; echo "loopback rc=$?"; tail -12 gpurun_out/pytest_loopback.log
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "dia_more or malformed or binding" > gpurun_out/pytest_robust.log 2>&1; echo "robust rc=$?"; tail -4 gpurun_out/pytest_robust.log
timeout 300 python tools/profile_variants.py --time c1 short > gpurun_out/variant_table_dia.json 2>/dev/null; echo "table rc=$?"
python -c "import json; t=json.load(open('gpurun_out/variant_table_dia.json')); [print(c, round(r['feature_ms'],3), {k: round(v['GBps']) for k,v in r['variants'].items()}) for c,r in t.items()]"
timeout 900 python bench.py > gpurun_out/bench_r02b.json 2> gpurun_out/bench_r02b.err; echo "bench rc=$?"
tail -30 gpurun_out/bench_r02b.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_r02b.json').read().strip().splitlines()[-1])
print({k: d[k] for k in ('value','ms_per_step','selected_variant','pct_of_exhaustive_best','bench_wall_s')})
print(d['roofline']); print(d['selection']); print(d.get('cpu_baseline')); print(d['e2e']); print(d['clocks'])
print({c: (v['picks'], v['exhaustive_best'], {k: round(e['GBps']) for k, e in v['exhaustive'].items()}) for c, v in d.get('configs', {}).items()})
sl = d.get('selection_leg', {}); print({k: (sl[k]['nitro_pct_mean'] if isinstance(sl.get(k), dict) and 'nitro_pct_mean' in sl[k] else sl.get(k)) for k in sl})
"
