"""Diagnostics: build a copy of libe3.so with one source recompiled under extra
defines (e.g. -DE3_GEMM_EXP=1) for same-box A/B runs through E3_LIB_PATH.
python scripts/build_variant.py OUT.so SOURCE.cu -DNAME=VALUE ..."""
import glob
import os
import subprocess
import sys

sys.path.insert(0, ".")
from paper_conf_sosp_iyergdpgn24_b200 import build as B  # noqa: E402

out, src, defs = sys.argv[1], sys.argv[2], sys.argv[3:]
B.build()
os.makedirs(os.path.dirname(os.path.abspath(out)), exist_ok=True)
obj_dir = os.path.join(B.ROOT, "build", "obj")
stem = os.path.splitext(os.path.basename(src))[0]
vobj = os.path.abspath(out) + "." + stem + ".o"
cmd = [B._nvcc(), *B.ARCH, *B.FLAGS, *defs, "-c", os.path.join(B.CSRC, src), "-o", vobj]
subprocess.run(cmd, check=True)
objs = [o for o in sorted(glob.glob(os.path.join(obj_dir, "*.o"))) if os.path.basename(o) != stem + ".o"
        and not os.path.basename(o).startswith(stem + ".")]
objs = [o for o in objs if os.path.splitext(os.path.basename(o))[0].split(".")[0] != stem]
subprocess.run([B._nvcc(), *B.ARCH, "-shared", "-o", out, *objs, vobj, "-ldl"], check=True)
print("built", out, "from", len(objs) + 1, "objects")
