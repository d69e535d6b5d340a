"""Build the library of a git ref as an A/B variant (no GPU needed).

usage: python tools/ab_ref.py <name> <git-ref>
-> paper_conf_sc_markidis23_b200/_variants/libsvb200_<name>.so; select it at
run time with SVB200_LIB=<that path> (the C ABI must match the current binding).
"""
import os
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_markidis23_b200 import build as B  # noqa: E402

name, ref = sys.argv[1], sys.argv[2]
tmp = tempfile.mkdtemp(prefix=f"ab_{name}_")
for sub in ("paper_conf_sc_markidis23_b200/csrc", "include"):
    os.makedirs(os.path.join(tmp, sub), exist_ok=True)
    files = subprocess.check_output(["git", "-C", ROOT, "ls-tree", "--name-only", f"{ref}:{sub}"], text=True).split()
    for f in files:
        data = subprocess.check_output(["git", "-C", ROOT, "show", f"{ref}:{sub}/{f}"])
        open(os.path.join(tmp, sub, f), "wb").write(data)
print(B.build_variant(name, [], csrc=os.path.join(tmp, "paper_conf_sc_markidis23_b200/csrc"),
                      include=os.path.join(tmp, "include")))
