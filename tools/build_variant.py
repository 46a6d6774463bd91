"""Build liblzr variants for A/B timing: python tools/build_variant.py NAME file.cu [-DX ...]
(file.cu replaces the csrc file of the same base name -- encode.cu unless the
name is one of csrc's -- in a temp copy; output paper_conf_pact_map17_b200/liblzr_NAME.so)"""
import os, shutil, subprocess, sys, tempfile
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_pact_map17_b200 import _build
name, enc = sys.argv[1], sys.argv[2]
extra = sys.argv[3:]
tmp = tempfile.mkdtemp()
src = os.path.join(tmp, "csrc")
shutil.copytree(_build.CSRC, src)
base = os.path.basename(enc)
shutil.copy(enc, os.path.join(src, base if os.path.exists(os.path.join(src, base)) else "encode.cu"))
inc = os.path.join(os.path.dirname(tmp), "include")
srcs = sorted(os.path.join(src, f) for f in os.listdir(src) if f.endswith(".cu"))
out = os.path.join(_build.PKG, f"liblzr_{name}.so")
# the sources include ../../include/lzr.h: mirror the layout
os.makedirs(os.path.join(tmp, "x", "y"), exist_ok=True)
shutil.move(src, os.path.join(tmp, "x", "y", "csrc"))
os.makedirs(os.path.join(tmp, "x", "include"), exist_ok=True)
shutil.copy(os.path.join(_build.ROOT, "include", "lzr.h"), os.path.join(tmp, "x", "include"))
srcs = sorted(os.path.join(tmp, "x", "y", "csrc", f) for f in os.listdir(os.path.join(tmp, "x", "y", "csrc")) if f.endswith(".cu"))
subprocess.check_call(["nvcc", *_build.NVCC_FLAGS, *extra, "-o", out, *srcs])
print(out)
