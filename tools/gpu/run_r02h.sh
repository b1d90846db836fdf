mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bench.py tests/test_gpu_parity.py -q -x -rf -k "bench or stream or impls" > gpurun_out/pytest_bench.log 2>&1; echo "rc=$?"; tail -8 gpurun_out/pytest_bench.log
timeout 900 python bench.py --dist --quick --no-cpu --steps 5 > gpurun_out/bench_dist1.json 2> gpurun_out/bench_dist1.err; echo "dist1 rc=$?"; tail -5 gpurun_out/bench_dist1.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_dist1.json').read().strip().splitlines()[-1]); print({k: d[k] for k in ('value','ms_per_step','selected_variant','pct_of_exhaustive_best')}); print(d.get('halo_exchange')); print(d['config']['parallelism'])"
