"""Build an experiment variant of libplgpu.so with extra nvcc defines into _variants/<name>.so
(load it with PLGPU_LIB=_variants/<name>.so).  usage: python tools/build_variant.py name -DX=1 ..."""
import importlib.util
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
spec = importlib.util.spec_from_file_location("_b", os.path.join(ROOT, "paper_conf_icppw_planob21_b200", "build.py"))
B = importlib.util.module_from_spec(spec)
spec.loader.exec_module(B)
name, defs = sys.argv[1], sys.argv[2:]
out = os.path.join(ROOT, "_variants")
os.makedirs(out, exist_ok=True)
objs = []
for src in B.SOURCES:
    obj = os.path.join(out, f"{name}_{src}.o")
    subprocess.run([B.NVCC, *B.ARCH, *B.FLAGS, *defs, "-c", os.path.join(B.CSRC, src), "-o", obj], check=True)
    objs.append(obj)
subprocess.run([B.NVCC, *B.ARCH, "-shared", "-o", os.path.join(out, name + ".so"), *objs, "-lcudart"], check=True)
for o in objs:
    os.remove(o)
print(os.path.join(out, name + ".so"))
