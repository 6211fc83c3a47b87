"""Same-box A/B builds: tools/_ablate/base/ holds a copy of the package whose library is compiled
from the csrc/ files of a git revision (default HEAD), so a working-tree change can be timed
against it in one gpurun call: MSORT_PKG_ROOT=tools/_ablate/base python tools/time_radix.py ...
usage: python tools/ab_build.py [REV]"""
import os, shutil, subprocess, sys, tempfile
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sigmod_maltenbergeritr22_b200 import build as b  # noqa: E402

rev = sys.argv[1] if len(sys.argv) > 1 else "HEAD"
dst = os.path.join(ROOT, "tools", "_ablate", "base", "paper_conf_sigmod_maltenbergeritr22_b200")
os.makedirs(os.path.join(dst, "_build"), exist_ok=True)
for f in os.listdir(b.HERE):
    if f.endswith(".py"):
        shutil.copy(os.path.join(b.HERE, f), dst)
tmp = tempfile.mkdtemp()
src_dir = os.path.join(tmp, "pkg", "csrc")  # csrc includes ../../include/msort.h
os.makedirs(src_dir)
os.makedirs(os.path.join(tmp, "include"))
with open(os.path.join(tmp, "include", "msort.h"), "wb") as fh:
    fh.write(subprocess.run(["git", "show", f"{rev}:include/msort.h"], cwd=ROOT, capture_output=True, check=True).stdout)
for f in b.SOURCES + b.HEADERS:
    data = subprocess.run(["git", "show", f"{rev}:paper_conf_sigmod_maltenbergeritr22_b200/csrc/{f}"], cwd=ROOT,
                          capture_output=True, check=True).stdout
    with open(os.path.join(src_dir, f), "wb") as fh:
        fh.write(data)
objs = []
for src in b.SOURCES:
    obj = os.path.join(dst, "_build", os.path.splitext(src)[0] + ".o")
    subprocess.run([b._nvcc(), *b.ARCH, *b.FLAGS, "-x", "cu", "-c", os.path.join(src_dir, src), "-o", obj], check=True)
    objs.append(obj)
subprocess.run([b._nvcc(), *b.ARCH, "-shared", "-cudart", "static", "-o", os.path.join(dst, "libmsort.so"), *objs,
                "-lpthread", "-ldl", "-lrt"], check=True)
print(dst)
