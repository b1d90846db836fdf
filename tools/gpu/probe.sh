# build and run one probe under tools/probes: bash tools/gpu/probe.sh <name>
mkdir -p gpurun_out
cd tools/probes && nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o $1 $1.cu && timeout 600 ./$1 | tee ../../gpurun_out/$1.jsonl
