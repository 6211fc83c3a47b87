"""Timing-ablation builds of libmsort (wrong results by design; never used by
tests or bench): tools/_ablate/<k>/ holds a copy of the package whose
library is compiled with -DMSORT_ABLATE=<k> (radix.cu: 1 = no look-back,
2 = no early counts, 3 = both), or, for a name of the form NAME=VALUE (e.g.
MSORT_LDHINT=1), with -DNAME=VALUE in tools/_ablate/NAME_VALUE/ (correct
results: a compile-time variant).  Time with MSORT_PKG_ROOT=tools/_ablate/<dir>."""
import os, shutil, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sigmod_maltenbergeritr22_b200 import build as b  # noqa: E402

for k in sys.argv[1:] or ["1", "2", "3"]:
    define = k if "=" in k else f"MSORT_ABLATE={k}"
    dst = os.path.join(ROOT, "tools", "_ablate", k.replace("=", "_"), "paper_conf_sigmod_maltenbergeritr22_b200")
    os.makedirs(os.path.join(dst, "_build"), exist_ok=True)
    for f in os.listdir(b.HERE):
        if f.endswith(".py"):
            shutil.copy(os.path.join(b.HERE, f), dst)
    objs = []
    for src in b.SOURCES:
        obj = os.path.join(dst, "_build", os.path.splitext(src)[0] + ".o")
        subprocess.run([b._nvcc(), *b.ARCH, *b.FLAGS, f"-D{define}", "-x", "cu", "-c",
                        os.path.join(b.CSRC, src), "-o", obj], check=True)
        objs.append(obj)
    subprocess.run([b._nvcc(), *b.ARCH, "-shared", "-cudart", "static", "-o", os.path.join(dst, "libmsort.so"), *objs,
                    "-lpthread", "-ldl", "-lrt"], check=True)
    print(dst)
