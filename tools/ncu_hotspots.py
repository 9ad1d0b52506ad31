"""Summarise an `ncu --page source --csv --print-source sass` export: stall samples by
reason, and the top instructions (with their stall mix)."""
import csv
import sys
from collections import Counter

rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
data = rows[2:]
isrc, iss = h.index("Source"), h.index("Warp Stall Sampling (All Samples)")
iex = h.index("Instructions Executed")
reasons = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
tot = Counter()
per = []
for r in data:
    try:
        s = int(r[iss] or 0)
    except ValueError:
        continue
    mix = {c: int(r[h.index(c)] or 0) for c in reasons}
    for c, v in mix.items():
        tot[c] += v
    per.append((s, r[isrc].strip(), int(r[iex] or 0), mix))
T = sum(tot.values())
print("total samples", T)
for c, v in tot.most_common():
    if v:
        print(f"  {c:24s} {v:8d} {100 * v / T:5.1f}%")
# group by opcode
op = Counter()
for s, src, ex, mix in per:
    op[src.split()[0] if not src.startswith("@") else src.split()[1]] += s
print("by opcode:")
for k, v in op.most_common(15):
    print(f"  {k:20s} {v:8d} {100 * v / T:5.1f}%")
print("top instructions:")
for s, src, ex, mix in sorted(per, key=lambda x: -x[0])[: int(sys.argv[2]) if len(sys.argv) > 2 else 25]:
    top = ", ".join(f"{k[6:]}={v}" for k, v in sorted(mix.items(), key=lambda x: -x[1])[:3] if v)
    print(f"  {s:7d} {src[:60]:60s} | {top}")
