# ncu full capture of chosen kernels on one config: CFG=c2b KREGEX='k_csr_vector|k_hyb_tail' VARS="csr_vector hyb"
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:${KREGEX}" -c ${COUNT:-4} \
    -o /tmp/kp_$CFG -f python tools/profile_variants.py $CFG $VARS > gpurun_out/kp_$CFG.log 2>&1
echo "ncu rc=$?"
ncu -i /tmp/kp_$CFG.ncu-rep --page details --csv > gpurun_out/kp_${CFG}_details.csv 2>/dev/null
ncu -i /tmp/kp_$CFG.ncu-rep --page raw --csv > gpurun_out/kp_${CFG}_raw.csv 2>/dev/null
for k in $SRCK; do
  ncu -i /tmp/kp_$CFG.ncu-rep --page source --csv -k regex:$k -c 1 > gpurun_out/kp_${CFG}_src_$k.csv 2>/dev/null
done
ls -la gpurun_out | grep kp_
