"""Opcode mix of a SASS address range: python tools/sass_mix.py file.sass START END"""
import re, sys, collections
txt = open(sys.argv[1]).read().splitlines()
lo, hi = int(sys.argv[2], 16), int(sys.argv[3], 16)
ALU = {"LOP3", "SHF", "IADD3", "ISETP", "SEL", "PLOP3", "LEA", "PRMT", "IABS", "IMNMX", "FLO", "SGXT", "LOP", "VIADD", "VIMNMX", "BMSK", "MOV", "P2R", "R2P"}
FMA = {"IMAD", "IMUL", "FFMA", "FMUL", "FADD"}
XU = {"POPC", "BREV", "MUFU"}
c = collections.Counter()
for line in txt:
    m = re.match(r"\s+/\*([0-9a-f]+)\*/\s+(@!?U?P[0-9T]\s+)?([A-Z0-9_]+)", line)
    if not m:
        continue
    a = int(m.group(1), 16)
    if lo <= a < hi:
        c[m.group(3)] += 1
tot = sum(c.values())
pipe = collections.Counter()
for k, v in c.items():
    pipe["alu" if k in ALU else "fma" if k in FMA else "xu" if k in XU else "other"] += v
print("total", tot, dict(pipe))
print(c.most_common(20))
