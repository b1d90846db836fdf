# predicated-gather batching (K6s hot, K9b HYB tail): ab/libnitro_head.so vs in-tree
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gather.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_gather.log
summ() { python -c "import json,sys; t=json.load(open(sys.argv[1])); print(' '.join(f'{c} '+' '.join(f'{k}:{v[\"ms\"]:.4f}' for k,v in r['variants'].items()) for c,r in t.items()))" $1; }
for rep in 1 2; do
  NITRO_LIB=$PWD/ab/libnitro_head.so timeout 600 python tools/profile_variants.py --time c2b c2a uvar3 band01 csr_vector hyb > gpurun_out/g_head.json 2>/dev/null; echo "head: $(summ gpurun_out/g_head.json)"
  timeout 600 python tools/profile_variants.py --time c2b c2a uvar3 band01 csr_vector hyb > gpurun_out/g_new.json 2>/dev/null; echo "new : $(summ gpurun_out/g_new.json)"
done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum --clock-control none --csv -k regex:'k_csr_stream|k_hyb_tail' -c 4 python tools/profile_variants.py c2b csr_vector hyb 2>/dev/null | grep -E 'k_csr_stream|k_hyb_tail' | awk -F'","' '{print substr($5,1,40), $(NF-2), $NF}'
