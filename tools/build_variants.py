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
    d = os.path.join(ROOT, "exp", name)
    if os.path.exists(d):
        shutil.rmtree(d)
    cs = os.path.join(d, "csrc")
    shutil.copytree(src or B.CSRC, cs)
    for fname, a, b in subs:
        p = os.path.join(cs, fname)
        t = open(p).read()
        assert a in t, (fname, a)
        open(p, "w").write(t.replace(a, b))
    return B.build(out=os.path.join(d, "libmapsm.so"), csrc=cs, extra=[f"-D{x}" for x in defines])


if __name__ == "__main__":
    for spec in sys.argv[1:]:
        name, _, defs = spec.partition(":")
        print(variant(name, [x for x in defs.split(",") if x]))
