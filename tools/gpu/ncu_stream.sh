mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k 'regex:k_(csr_stream|hyb_tail_ls)' -c 2 \
   -o /tmp/prof_stream -f python tools/profile_variants.py c2b csr_vector hyb > gpurun_out/prof_stream.log 2>&1
echo "ncu rc=$?"
ncu -i /tmp/prof_stream.ncu-rep --page raw --csv > gpurun_out/prof_stream_raw.csv 2>/dev/null
ncu -i /tmp/prof_stream.ncu-rep --page source --csv -k regex:k_csr_stream -c 1 > gpurun_out/prof_stream_src.csv 2>/dev/null
ncu -i /tmp/prof_stream.ncu-rep --page details --csv > gpurun_out/prof_stream_details.csv 2>/dev/null
ls -la gpurun_out/prof_stream*
