# registers / spills per kernel instantiation of one source: bash tools/regs.sh spmv [filter]
cd "$(dirname "$0")/../paper_conf_ipps_muralidharanshgc14_b200"
nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -Xcompiler -fPIC -I ../include -Xptxas -v -c csrc/$1.cu -o /tmp/$1.o 2>&1 \
 | grep -E "Compiling entry|registers|spill" | paste - - - \
 | sed -E "s/.*entry function '([^']*)'.* ([0-9]+) bytes spill stores.*Used ([0-9]+) registers.*/\1 spill=\2 regs=\3/" \
 | c++filt | sed -E 's/\(anonymous namespace\):://; s/nitro:://g; s/\(.*\)//' | grep -E "${2:-.}"
