#!/usr/bin/env python
"""A/B builds: libnitro.so variants with extra nvcc defines for one source.

  python tools/ab_build.py NAME SRC.cu -DFOO=1 ...   ->  ab/libnitro_NAME.so
(the other objects come from the in-tree build; run build() first)"""
import os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "paper_conf_ipps_muralidharanshgc14_b200"))
import build as nb  # noqa: E402

name, src, defs = sys.argv[1], sys.argv[2], sys.argv[3:]
nb.build()
nccl = nb.nccl_dir()
os.makedirs(os.path.join(ROOT, "ab"), exist_ok=True)
obj = os.path.join(ROOT, "ab", f"{name}_{src}.o")
cmd = ["nvcc", "-O3", "-std=c++17", "-lineinfo", *nb.ARCH, "-Xcompiler", "-fPIC,-ffp-contract=off",
       "-I", nb.INCLUDE, "-I", os.path.join(nccl, "include"), *defs, "-c", os.path.join(nb.CSRC, src), "-o", obj]
subprocess.run(cmd, check=True)
objs = [obj if os.path.basename(s) == src else os.path.join(nb.OBJ, os.path.basename(s) + ".o") for s in nb._sources()]
so = os.path.join(ROOT, "ab", f"libnitro_{name}.so")
nlib = os.path.join(nccl, "lib")
subprocess.run(["nvcc", "-shared", *nb.ARCH, "-o", so, *objs, "-L", nlib, "-l:libnccl.so.2", "-Xlinker",
                f"-rpath,{nlib}"], check=True)
print(so)
