mkdir -p gpurun_out
timeout 1200 ncu --set full --clock-control none --import-source on -k 'regex:k_(features|dia)' -c 8 \
    -o /tmp/prof_c4 -f python tools/profile_variants.py c4 > gpurun_out/prof_c4.log 2>&1; echo "ncu c4 rc=$?"
ncu -i /tmp/prof_c4.ncu-rep --page raw --csv > gpurun_out/prof_c4_raw.csv 2>/dev/null
ncu -i /tmp/prof_c4.ncu-rep --page source --csv -k regex:k_dia -c 1 > gpurun_out/prof_c4_src_dia.csv 2>/dev/null
for i in 1 2; do timeout 600 python tools/e2e_chunks.py 16 2>&1 | tail -1; done; nvidia-smi -q | grep -i -A3 "PCIe Generation\|Link Width" | head -12
