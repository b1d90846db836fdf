python tools/hist_probe.py --time uniform; python tools/hist_probe.py --time spike; python tools/hist_probe.py --time normal
timeout 900 ncu --set full --clock-control none -k 'regex:k_hist_(shared|global|sort)' -c 12 -o /tmp/prof_hist -f python tools/hist_probe.py uniform > gpurun_out/prof_hist.log 2>&1; echo "ncu rc=$?"
ncu -i /tmp/prof_hist.ncu-rep --page raw --csv > gpurun_out/prof_hist_raw.csv 2>/dev/null
ls -la gpurun_out/prof_hist_raw.csv
