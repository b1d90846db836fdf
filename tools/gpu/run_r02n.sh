mkdir -p gpurun_out
timeout 900 python tools/profile_variants.py --time band48 band96h c1big short band01 uvar3 > gpurun_out/variant_classes.json 2>/dev/null; echo "rc=$?"
python -c "import json; t=json.load(open('gpurun_out/variant_classes.json')); [print(c, r['rows'], r['nnz'], {k: (round(v['GBps']), round(v['ms'],4)) for k,v in r['variants'].items()}) for c,r in t.items()]"
timeout 300 python bench.py --gpus 2 --quick --no-cpu --steps 3 > gpurun_out/bench_gpus2.out 2> gpurun_out/bench_gpus2.err; echo "gpus2 rc=$?"; cat gpurun_out/bench_gpus2.out; tail -3 gpurun_out/bench_gpus2.err
