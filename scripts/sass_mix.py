#!/usr/bin/env python3
"""Static SASS instruction mix of the hot kernels (cuobjdump -sass of build/kernels.o).

    python scripts/sass_mix.py [build/kernels.o] > profiles/r02/sass_mix.md

Per kernel instantiation: instruction count and the opcodes that show what the kernel does --
the 256/128-bit streaming loads (LDG ... .NA = L1::no_allocate, .ENL2 = L2 cache-hint), the x
gathers (LDG.E.CONSTANT = ld.global.nc), the tensor-core block dots (DMMA / HMMA), CUDA-core FMAs,
shuffles, y stores, and local-memory spills (LDL / STL).  Template arguments: <dtype, variant>,
dtype 0 FP64 / 1 FP16 / 2 FP32; variant 1 MMA / 2 CUDA-core, +4 = scatter epilogue.
"""
import collections
import re
import subprocess
import sys

obj = sys.argv[1] if len(sys.argv) > 1 else "build/kernels.o"
sass = subprocess.run(["cuobjdump", "-sass", obj], capture_output=True, text=True, check=True).stdout

funcs = collections.OrderedDict()
cur = None
for line in sass.splitlines():
    m = re.search(r"Function : (\S+)", line)
    if m:
        cur = m.group(1)
        funcs[cur] = []
        continue
    m = re.match(r"\s+/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]*)", line)
    if m and cur:
        funcs[cur].append(m.group(1))


def short(name):
    m = re.search(r"(dasp_\w+?_kernel)I(.*?)E+v", name)
    if not m:
        m2 = re.search(r"(dasp_\w+?_kernel)", name)
        return m2.group(1) if m2 else name
    args = re.findall(r"Li(\d+)E", m.group(2) + "E")
    return f"{m.group(1)}<{','.join(args)}>" if args else f"{m.group(1)}<{m.group(2)}>"


COLS = [
    ("instr", lambda op: True),
    ("LDG 256b", lambda op: op.startswith("LDG") and ".256" in op),
    ("LDG 128b", lambda op: op.startswith("LDG") and ".128" in op),
    ("LDG .NA (no L1 alloc)", lambda op: op.startswith("LDG") and ".NA" in op),
    ("LDG.CONSTANT (x gathers)", lambda op: op.startswith("LDG") and "CONSTANT" in op),
    ("LDG other", lambda op: op.startswith("LDG") and ".NA" not in op and "CONSTANT" not in op),
    ("STG", lambda op: op.startswith("STG")),
    ("DMMA", lambda op: op.startswith("DMMA")),
    ("HMMA", lambda op: op.startswith("HMMA")),
    ("DFMA", lambda op: op.startswith("DFMA")),
    ("FFMA", lambda op: op.startswith("FFMA")),
    ("SHFL", lambda op: op.startswith("SHFL")),
    ("UBLKCP/UTMALDG", lambda op: op.startswith("UBLKCP") or op.startswith("UTMALDG")),
    ("LDL/STL (spill)", lambda op: op.startswith("LDL") or op.startswith("STL")),
]

print("# SASS instruction mix (static counts, `cuobjdump -sass build/kernels.o`)\n")
print("Template arguments `<dtype, variant>`: dtype 0 FP64, 1 FP16, 2 FP32; variant 1 MMA, 2 CUDA-core, "
      "+4 scatter epilogue (dasp_spmv_scatter).  `.NA` = `ld.global.nc.L1::no_allocate` streams with an L2 "
      "cache-hint policy (evict_first); `LDG.E.CONSTANT` = x gathers through the read-only path.\n")
print("| kernel | " + " | ".join(c for c, _ in COLS) + " |")
print("|---|" + "---|" * len(COLS))
for name, ops in funcs.items():
    if "dasp_main_kernel" not in name and "dasp_long_kernel" not in name:
        continue
    cnt = [sum(1 for op in ops if f(op)) for _, f in COLS]
    print(f"| `{short(name)}` | " + " | ".join(str(c) for c in cnt) + " |")
print("\nMost frequent load / store / tensor opcodes per kernel (full mnemonic):\n")
for name, ops in funcs.items():
    if "dasp_main_kernel" not in name and "dasp_long_kernel" not in name:
        continue
    c = collections.Counter(op for op in ops if op.startswith(("LDG", "STG", "DMMA", "HMMA", "LDL", "STL")))
    print(f"* `{short(name)}`: " + ", ".join(f"{k} x{v}" for k, v in c.most_common(8)))
