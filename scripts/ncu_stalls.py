"""Stall-reason totals of an ncu report restricted to an address range and execution count band."""
import csv, io, subprocess, sys
rep, lo, hi = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
a0 = int(sys.argv[4], 16) if len(sys.argv) > 4 else 0
a1 = int(sys.argv[5], 16) if len(sys.argv) > 5 else 1 << 62
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[1]; data = rows[2:]
iex = h.index("Instructions Executed")
cols = [i for i, x in enumerate(h) if x.startswith("stall_") and "Not Issued" not in x]
tot = {h[i]: 0 for i in cols}
n = 0; ex = 0
for x in data:
    e = int(x[iex] or 0)
    a = int(x[0], 16) & 0xFFFFF
    if lo <= e <= hi and a0 <= a < a1:
        n += 1; ex += e
        for i in cols: tot[h[i]] += int(x[i] or 0)
s = sum(tot.values())
print(f"{n} instructions, {s} samples")
for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
    if v: print(f"  {k:28s} {v:8d} {100*v/s:5.1f}%")
