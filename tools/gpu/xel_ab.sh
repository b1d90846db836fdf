# c2b CSR-vector (K6s hot) with evict_last x gathers (ab/libnitro_xel.so) vs the in-tree build
mkdir -p gpurun_out
summ() { python -c "import json,sys; t=json.load(open(sys.argv[1])); print(' '.join(f'{c} '+' '.join(f'{k}:{v[\"ms\"]:.4f}' for k,v in r['variants'].items()) for c,r in t.items()))" $1; }
for rep in 1 2 3; do
  for lib in xel; do
    NITRO_LIB=$PWD/ab/libnitro_$lib.so timeout 600 python tools/profile_variants.py --time ${CF:-c2b} ${VARS:-csr_vector} > gpurun_out/xel_$lib.json 2>/dev/null; echo "$lib: $(summ gpurun_out/xel_$lib.json)"
  done
  timeout 600 python tools/profile_variants.py --time ${CF:-c2b} ${VARS:-csr_vector} > gpurun_out/xel_new.json 2>/dev/null; echo "new: $(summ gpurun_out/xel_new.json)"
done
for lib in xel new; do
  L=$PWD/ab/libnitro_$lib.so; [ $lib = new ] && L=$PWD/paper_conf_ipps_muralidharanshgc14_b200/libnitro.so
  NITRO_LIB=$L timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum --clock-control none --csv -k regex:k_csr_stream -c 2 python tools/profile_variants.py c2b csr_vector 2>/dev/null | grep -E 'k_csr_stream' | awk -F'","' '{print "'$lib'", $(NF-2), $(NF-1), $NF}' | tail -6
done
