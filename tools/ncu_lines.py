"""Per-CUDA-source-line stall samples from `ncu --page source --csv --print-source cuda,sass`.
usage: python tools/ncu_lines.py export.csv [top=40] [first_line] [last_line]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Line No")
h = rows[hi]
iss = h.index("Warp Stall Sampling (All Samples)")
iex = h.index("Instructions Executed")
reasons = [(i, c) for i, c in enumerate(h) if c.startswith("stall_") and "Not Issued" not in c]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
lo = int(sys.argv[3]) if len(sys.argv) > 3 else 0
up = int(sys.argv[4]) if len(sys.argv) > 4 else 10 ** 9
lines = []
for r in rows[hi + 1:]:
    if r and r[0] and r[0].isdigit():
        ln = int(r[0])
        try:
            s = int(r[iss] or 0)
        except ValueError:
            continue
        if not (lo <= ln <= up):
            continue
        mix = sorted(((int(r[i] or 0), c[6:]) for i, c in reasons), reverse=True)[:3]
        lines.append((s, ln, r[1].strip(), int(r[iex] or 0), mix))
T = sum(x[0] for x in lines)
print("samples in range", T)
for s, ln, src, ex, mix in sorted(lines, reverse=True)[:top]:
    print(f"{100 * s / T:5.1f}% L{ln:4d} inst {ex:>12d} {src[:70]:70s} | " + ", ".join(f"{c}={v}" for v, c in mix if v))
