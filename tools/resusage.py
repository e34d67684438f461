#!/usr/bin/env python
"""Registers / shared memory / stack per kernel of a cubin-bearing object (cuobjdump -res-usage).
usage: python tools/resusage.py file.o|.so [regex]"""
import re, subprocess, sys
out = subprocess.run(["cuobjdump", "-res-usage", sys.argv[1]], capture_output=True, text=True).stdout
pat = re.compile(sys.argv[2]) if len(sys.argv) > 2 else None
lines = out.splitlines()
for i, l in enumerate(lines):
    m = re.match(r"\s*Function (\S+):", l)
    if not m:
        continue
    name = subprocess.run(["c++filt", m.group(1)], capture_output=True, text=True).stdout.strip()
    name = re.sub(r"\(.*", "", name)
    res = lines[i + 1].strip()
    r = dict(re.findall(r"(\w+):(\d+)", res))
    if pat and not pat.search(name):
        continue
    print(f"{name[:100]:100s} REG={r.get('REG')} STACK={r.get('STACK')} SHARED={r.get('SHARED')}")
