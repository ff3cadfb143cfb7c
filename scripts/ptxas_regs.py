"""Registers and spills per kernel from the in-tree build's ptxas logs.

    python scripts/ptxas_regs.py [SUBSTRING] [FILE-STEM]
"""
import glob
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sub = sys.argv[1] if len(sys.argv) > 1 else ""
stem = sys.argv[2] if len(sys.argv) > 2 else "*"
pat = re.compile(r"Compiling entry function '(\S+)'[^\n]*\n[^\n]*\n\s*(\d+) bytes stack frame, (\d+) bytes spill stores, "
                 r"(\d+) bytes spill loads\n[^\n]*Used (\d+) registers")
for f in sorted(glob.glob(os.path.join(ROOT, "paper_conf_icpp_nagasakanm17_b200", "_build", stem + ".o.ptxas.log"))):
    for m in pat.finditer(open(f).read()):
        if sub in m.group(1):
            print(f"{m.group(5):>4} regs  spill {m.group(3):>4}/{m.group(4):<4} {m.group(1)[:110]}")
