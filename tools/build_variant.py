"""Build an ablation variant of libharmonia.so with extra -D macros into tools/bin/<name>.so
(run with HARMONIA_LIB=tools/bin/<name>.so; tools/bin travels with gpurun).  Used only for A/B measurements.

    python tools/build_variant.py NAME [-DMACRO[=V] ...]
"""
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_yanlpz19_b200 import _build as b  # noqa: E402

name, defs = sys.argv[1], sys.argv[2:]
out_dir = os.path.join(b.ROOT, "tools", "bin")
tmp = os.path.join(out_dir, "obj_" + name)
os.makedirs(tmp, exist_ok=True)
procs, objs = [], []
for s in b.sources():
    o = os.path.join(tmp, os.path.basename(s) + ".o")
    objs.append(o)
    cmd = [b.nvcc(), "-c", s, "-o", o] + [f for f in b.NVCC_FLAGS if f != "-shared"] + defs
    procs.append(subprocess.Popen(cmd))
if any(p.wait() for p in procs):
    sys.exit("nvcc failed")
subprocess.check_call([b.nvcc(), "-shared", "-Xcompiler", "-fPIC", "-gencode", "arch=compute_100a,code=sm_100a",
                       "-o", os.path.join(out_dir, name + ".so")] + objs)
print(os.path.join(out_dir, name + ".so"))
