"""Build an experimental variant of libpesto.so with extra nvcc -D flags for eval32.cu.

usage: python scripts/build_variant.py NAME -DPESTO_E32_STAGES=2 -DPESTO_E32_MINB2=4 ...
writes paper_conf_middleware_hafeezsg021_b200/libpesto_NAME.so (load it with PESTO_LIB=...).
VARSRC=kernels.cu,eval32.cu recompiles those translation units with the flags (default eval32.cu).
"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_middleware_hafeezsg021_b200")
sys.path.insert(0, ROOT)
from paper_conf_middleware_hafeezsg021_b200 import build as B  # noqa: E402

B.build()
name, defs = sys.argv[1], sys.argv[2:]
bdir = os.path.join(B.BUILD, "var_" + name)
os.makedirs(bdir, exist_ok=True)
varsrc = os.environ.get("VARSRC", "eval32.cu").split(",")
vobj = {}
for f in varsrc:
    o = os.path.join(bdir, f + ".o")
    src = (os.environ.get("SRC32") if f == "eval32.cu" else None) or os.path.join(B.CSRC, f)
    subprocess.run([B.NVCC, *B.ARCH, "-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC",
                    *defs, "-Xptxas", "-v", "-I", B.INC, "-I", B.CSRC, "-c", src, "-o", o],
                   check=True, capture_output=True)
    vobj[f] = o
objs = [vobj.get(f, os.path.join(B.BUILD, f + ".o")) for f in B.CU_SOURCES + B.CPP_SOURCES]
out = os.path.join(PKG, f"libpesto_{name}.so")
subprocess.run([B.NVCC, *B.ARCH, "-shared", "-cudart", "static", "-o", out, *objs, "-ldl",
                "-lpthread", "-lrt"], check=True)
print(out)
