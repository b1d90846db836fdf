mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k 'regex:k_csr_stream' -c 1 \
   -o /tmp/prof_hot -f python tools/profile_variants.py c2b csr_vector > gpurun_out/prof_hot.log 2>&1
echo "ncu rc=$?"
ncu -i /tmp/prof_hot.ncu-rep --page raw --csv > gpurun_out/prof_hot_raw.csv 2>/dev/null
ncu -i /tmp/prof_hot.ncu-rep --page source --csv -k regex:k_csr_stream -c 1 > gpurun_out/prof_hot_src.csv 2>/dev/null
ls -la gpurun_out/prof_hot*
