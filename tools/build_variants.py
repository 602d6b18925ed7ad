"""Build kernel-tuning variants of libmapsm into exp/<name>/ (git-ignored).

Each variant = the in-tree csrc/ with optional text substitutions and extra
nvcc flags.  Usage: python tools/build_variants.py name:FLAG=..[,...] ..."""
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_ben_nunlbr15_b200 import build as B  # noqa: E402


def variant(name, defines=(), subs=(), src=None):
    """Only the translation units that mention a defined macro (or carry a
    substitution) are recompiled; the others reuse the in-tree objects."""
    d = os.path.join(ROOT, "exp", name)
    if os.path.exists(d):
        shutil.rmtree(d)
    cs = os.path.join(d, "csrc")
    shutil.copytree(src or B.CSRC, cs)
    shutil.copytree(B.OBJ, os.path.join(d, "_build"))  # copy2: mtimes kept
    touched = set()
    for fname, a, b in subs:
        p = os.path.join(cs, fname)
        t = open(p).read()
        assert a in t, (fname, a)
        open(p, "w").write(t.replace(a, b))
        touched.add(fname)
    macros = [x.split("=")[0] for x in defines]
    text = {f: open(os.path.join(cs, f)).read() for f in os.listdir(cs)}
    marked = {f for f, t in text.items() if any(m in t for m in macros)}
    for _ in range(3):  # files including a marked header (transitively)
        marked |= {f for f, t in text.items() if any(f'"{h}"' in t for h in marked if not h.endswith((".cu", ".cpp")))}
    touched |= {f for f in marked if f.endswith((".cu", ".cpp"))}
    import time
    now = time.time() + 1
    for fname in touched:
        os.utime(os.path.join(cs, fname), (now, now))
    out = B.build(out=os.path.join(d, "libmapsm.so"), csrc=cs, extra=[f"-D{x}" for x in defines])
    # only the library travels to the GPU box
    shutil.rmtree(cs)
    shutil.rmtree(os.path.join(d, "_build"))
    return out


if __name__ == "__main__":
    for spec in sys.argv[1:]:
        name, _, defs = spec.partition(":")
        print(variant(name, [x for x in defs.split(",") if x]))
