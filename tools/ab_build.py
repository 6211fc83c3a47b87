"""Same-box A/B builds: tools/_ablate/<name>/ holds a copy of the package whose library is compiled
from the csrc/ files of a git revision (REV, default HEAD) or of the working tree (REV = "WT"), with
optional extra nvcc defines, so variants can be timed against each other in one gpurun call:
MSORT_PKG_ROOT=tools/_ablate/<name> python tools/time_radix.py ...
usage: python tools/ab_build.py [REV|WT] [NAME] [-DFOO=...]..."""
import os, shutil, subprocess, sys, tempfile
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sigmod_maltenbergeritr22_b200 import build as b  # noqa: E402

rev = sys.argv[1] if len(sys.argv) > 1 else "HEAD"
name = sys.argv[2] if len(sys.argv) > 2 else "base"
defines = [a for a in sys.argv[3:] if a.startswith(("-D", "-X"))]  # defines and -Xptxas options
dst = os.path.join(ROOT, "tools", "_ablate", name, "paper_conf_sigmod_maltenbergeritr22_b200")
os.makedirs(os.path.join(dst, "_build"), exist_ok=True)
tmp = tempfile.mkdtemp()
src_dir = os.path.join(tmp, "pkg", "csrc")  # csrc includes ../../include/msort.h
os.makedirs(src_dir)
os.makedirs(os.path.join(tmp, "include"))


def read(path):
    if rev == "WT":
        with open(os.path.join(ROOT, path), "rb") as fh:
            return fh.read()
    return subprocess.run(["git", "show", f"{rev}:{path}"], cwd=ROOT, capture_output=True, check=True).stdout


for f in ("__init__.py", "build.py", "dist.py"):  # the binding of the same revision
    try:
        data = read(f"paper_conf_sigmod_maltenbergeritr22_b200/{f}")
    except subprocess.CalledProcessError:
        continue
    with open(os.path.join(dst, f), "wb") as fh:
        fh.write(data)
with open(os.path.join(tmp, "include", "msort.h"), "wb") as fh:
    fh.write(read("include/msort.h"))
for f in b.SOURCES + b.HEADERS:
    with open(os.path.join(src_dir, f), "wb") as fh:
        fh.write(read(f"paper_conf_sigmod_maltenbergeritr22_b200/csrc/{f}"))
objs = []
flags = [f for f in b.FLAGS]
flags[flags.index("-I") + 1] = os.path.join(tmp, "include")
for src in b.SOURCES:
    obj = os.path.join(dst, "_build", os.path.splitext(src)[0] + ".o")
    subprocess.run([b._nvcc(), *b.ARCH, *flags, *defines, "-x", "cu", "-c", os.path.join(src_dir, src), "-o", obj],
                   check=True)
    objs.append(obj)
subprocess.run([b._nvcc(), *b.ARCH, "-shared", "-cudart", "static", "-o", os.path.join(dst, "libmsort.so"), *objs,
                *b.LINK_LIBS], check=True)
print(dst)
