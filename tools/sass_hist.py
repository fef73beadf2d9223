"""Instruction mix of one draw of the default bulk-fill kernel (tool).

    python tools/sass_hist.py > profiles/r01_fill_sass.txt
Reads the SASS of libggprng.so (cuobjdump), finds the first mbarrier wait of
the x2 fill kernel's draw loop and counts the instructions up to the next one
(= one draw of two walkers = 2 labels).
"""
import collections
import os
import re
import subprocess

LIB = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                   "paper_conf_ipps_banerjeebk12_b200", "libggprng.so")
KERNEL = "_ZN2gg21gg_fill64t_tma_kernelILi4ELi0ELb1ELb0ELb1EEEv14CUtensorMap_stNS_8FillArgsEjPj"
ALU = ("LOP3", "SHF", "LEA", "IADD3", "R2P", "ISETP", "SEL", "PLOP3", "VIADD", "MOV", "LOP")

out = subprocess.run(["cuobjdump", "-sass", LIB], capture_output=True, text=True, check=True).stdout
body = None
for f in re.split(r"\n\s+Function : ", out):
    if f.startswith(KERNEL):
        body = f
ins = [t for _, t in re.findall(r"/\*([0-9a-f]{4})\*/\s+([^;]*);", body)]
waits = [i for i, t in enumerate(ins) if "TRYWAIT" in t]
seg = ins[waits[0]:waits[1]]
h = collections.Counter()
for t in seg:
    tok = t.split()
    h[tok[1] if tok[0].startswith("@") else tok[0]] += 1
tot = sum(h.values())
heavy = sum(v for k, v in h.items() if k.startswith("IMAD"))
alu = sum(v for k, v in h.items() if k.split(".")[0] in ALU)
print(f"{KERNEL}: one draw of two walkers (2 labels), {tot} SASS = {tot / 2:.1f} per label")
print(f"FMA-heavy (IMAD*) {heavy}, ALU {alu}, other {tot - heavy - alu}")
for k, v in h.most_common():
    print(f"{v:5d} {k}")
