#!/usr/bin/env python
"""Registers / spills per kernel instance from build/*.ptxas.log (nvcc -Xptxas -v).

    python scripts/ptxas_regs.py build/k_split.ptxas.log k_splitILi0ELi1ELi4ELi0E
"""
import re
import sys

cur = None
out = {}
for line in open(sys.argv[1]):
    m = re.search(r"Compiling entry function '(\S+)'", line)
    if m:
        cur = m.group(1)
        continue
    if cur is None:
        continue
    m = re.search(r"(\d+) bytes stack frame, (\d+) bytes spill stores, (\d+) bytes spill loads", line)
    if m:
        out.setdefault(cur, {})["spill"] = int(m.group(2))
    m = re.search(r"Used (\d+) registers", line)
    if m:
        out.setdefault(cur, {})["regs"] = int(m.group(1))
pats = sys.argv[2:] or [""]
for k, v in out.items():
    if any(p in k for p in pats):
        print(f"{v.get('regs')}\t{v.get('spill')}\t{k[:90]}")
