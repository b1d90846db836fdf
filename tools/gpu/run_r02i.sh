mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_c4.py tests/test_gpu_dist_loopback.py -q -x -rf -k "feature or canonical or c4 or loopback_ranks" > gpurun_out/pytest_feat.log 2>&1; echo "rc=$?"; tail -4 gpurun_out/pytest_feat.log
timeout 600 python tools/profile_variants.py --time c1 c2a c2b uvar3 band01 short c4 none > gpurun_out/feat_new.json 2>/dev/null
python -c "import json; t=json.load(open('gpurun_out/feat_new.json')); [print(c, round(r['feature_ms'],3), round(r['feature_GBps'])) for c,r in t.items()]"
timeout 900 python bench.py --dist --quick --no-cpu --steps 5 > gpurun_out/bench_dist1.json 2> gpurun_out/bench_dist1.err; echo "dist1 rc=$?"; tail -3 gpurun_out/bench_dist1.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_dist1.json').read().strip().splitlines()[-1]); print({k: d[k] for k in ('value','ms_per_step','selected_variant','pct_of_exhaustive_best')}); print(d.get('halo_exchange')); print(d['config']['parallelism']); print(d['exhaustive'])"
