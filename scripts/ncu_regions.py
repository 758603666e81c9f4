"""Warp-stall samples of an ncu report split into the kernel's regions: the steady 16-step block
(the longest straight run with 16 STS.128), the rest of the compute warp, helper warps; per-region
stall reasons.  python scripts/ncu_regions.py rep.ncu-rep"""
import csv, io, subprocess, collections, sys
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = [i for i, r in enumerate(rows) if r and r[0] == "Address"][0]
h = rows[hi]; data = [r for r in rows[hi + 1:] if len(r) > 5]
i_s = h.index("Warp Stall Sampling (All Samples)"); i_src = h.index("Source"); i_ex = h.index("Instructions Executed")
stall = [i for i, x in enumerate(h) if x.startswith("stall_") and "Not Issued" not in x]
num = lambda x: int(x) if x.isdigit() else 0
sts = [k for k, r in enumerate(data) if "STS.128" in r[i_src]]
best = None
for a in range(len(sts)):
    for b in range(a + 15, len(sts)):
        if sts[b] - sts[a] < 600 and b - a == 15:
            if best is None or sts[b] - sts[a] < best[1] - best[0]:
                best = (sts[a], sts[b])
lo, hi2 = best[0] - 30, best[1] + 20
def summ(sel, name):
    agg = collections.Counter(); s = 0; ex = 0
    for r in sel:
        s += num(r[i_s])
        for i in stall: agg[h[i][6:]] += num(r[i])
    print(f"{name:14s} samples {s:7d}  " + " ".join(f"{k}:{v}" for k, v in agg.most_common(8)))
summ(data[lo:hi2], "steady block")
summ(data[:lo] + data[hi2:], "rest")
print("steady block instructions", hi2 - lo, "executions of its first STS.128:", data[best[0]][i_ex])
