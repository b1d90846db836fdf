# pipelined run_host: e2e by chunk count
mkdir -p gpurun_out
for c in 1 4 8 16; do
  echo "RUN_HOST_CHUNKS=$c"
  NITRO_RUN_HOST_CHUNKS=$c timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu > gpurun_out/b_$c.json 2> gpurun_out/b_$c.err
  tail -3 gpurun_out/b_$c.err
  python -c "import json,sys; d=json.loads(open('gpurun_out/b_$c.json').read().strip().splitlines()[-1]); print(round(d['value']), d['e2e'], d['roofline'].get('size_matched_copy_gbs'), d['roofline'].get('frac_of_size_matched_copy'))"
done
