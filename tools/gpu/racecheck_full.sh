mkdir -p gpurun_out
for part in single single loopback loopback; do
NITRO_CSRV_HOT=2 SANITIZE_PARTS=$part timeout 1500 compute-sanitizer --tool racecheck --racecheck-report all python tools/sanitize_run.py > gpurun_out/racecheck_$part.txt 2>&1
echo "part $part"; grep -n -B2 -A14 "Error\|Hazard\|hazard\|Internal\|complete" gpurun_out/racecheck_$part.txt | head -30
done
