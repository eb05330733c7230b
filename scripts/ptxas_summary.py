"""Registers / spills per kernel instantiation from an nvcc -Xptxas -v log (build/kernels.ptxas.txt)."""
import re
import sys

cur = sp = None
for line in open(sys.argv[1] if len(sys.argv) > 1 else "build/kernels.ptxas.txt"):
    m = re.search(r"Compiling entry function '(\S+)'", line)
    if m:
        n = m.group(1)
        k = re.search(r"(dasp_\w+?_kernel)I((?:Li\d+E)+)", n)
        cur = f"{k.group(1)}<{','.join(re.findall(r'Li(\d+)E', k.group(2)))}>" if k else n[:60]
        continue
    m = re.search(r"(\d+) bytes spill stores, (\d+) bytes spill loads", line)
    if m and cur:
        sp = f"spill {m.group(1)}/{m.group(2)}"
        continue
    m = re.search(r"Used (\d+) registers", line)
    if m and cur:
        print(f"{cur:32s} regs {m.group(1):>3s}  {sp}")
        cur = None
