"""Summarise registers / smem / spills per kernel from build/ptxas.log."""
import os
import re
import subprocess
import sys

log = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                   "paper_conf_ipps_nisassvs18_b200", "build", "ptxas.log")
pat = sys.argv[1] if len(sys.argv) > 1 else ""
cur = None
spill = ""
for line in open(log).read().splitlines():
    m = re.search(r"Compiling entry function '(\S+)'", line)
    if m:
        cur = m.group(1)
        continue
    m = re.search(r"(\d+) bytes spill stores", line)
    if m:
        spill = m.group(1)
    m = re.search(r"Used (\d+) registers(.*)", line)
    if m and cur:
        dn = subprocess.run(["c++filt", cur], capture_output=True, text=True).stdout.strip()
        short = dn.split("::")[-1].split("(")[0]
        if pat in short:
            print(f"{short:60s} regs={m.group(1):>3s} spill={spill:>3s} {m.group(2).strip()}")
        cur = None
