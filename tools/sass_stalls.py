"""Decode the fixed-latency stall counts ptxas encoded in SASS (Volta+ control bits) for the
instructions between two markers, to estimate the single-warp cycle count of a loop body.
usage: cuobjdump -sass lib.so | python tools/sass_stalls.py FUNC_SUBSTR START_OPCODE_INDEX COUNT"""
import re
import sys

lines = sys.stdin.read().split("\n")
func = sys.argv[1]
infn = False
insts = []
i = 0
while i < len(lines):
    l = lines[i]
    if "Function :" in l:
        infn = func in l
    if infn:
        m = re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+(.*?);\s+/\* (0x[0-9a-f]+) \*/", l)
        if m and i + 1 < len(lines):
            m2 = re.search(r"/\* (0x[0-9a-f]+) \*/", lines[i + 1])
            hi = int(m2.group(1), 16)
            stall = (hi >> 41) & 0xF
            yld = (hi >> 45) & 1
            wbar = (hi >> 46) & 7
            rbar = (hi >> 49) & 7
            wait = (hi >> 52) & 0x3F
            insts.append((m.group(1), m.group(2).strip(), stall, yld, wbar, rbar, wait))
    i += 1
start = int(sys.argv[2]) if len(sys.argv) > 2 else 0
cnt = int(sys.argv[3]) if len(sys.argv) > 3 else len(insts)
tot = 0
for a, s, st, y, wb, rb, w in insts[start:start + cnt]:
    tot += st
    print(f"{a} st={st:2d} y={y} wb={wb} rb={rb} wait={w:06b}  {s[:70]}")
print("instructions", len(insts[start:start + cnt]), "sum of stall counts", tot)
