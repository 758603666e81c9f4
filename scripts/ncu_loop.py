"""Dump the SASS of the hottest loop body (instructions sharing one execution count) with
warp-stall samples from an ncu report:  python scripts/ncu_loop.py rep.ncu-rep [count]"""
import collections, csv, io, subprocess, sys
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
while rows and "Address" not in rows[0]:
    rows = rows[1:]
h, data = rows[0], rows[1:]
i_s = h.index("Warp Stall Sampling (All Samples)"); i_src = h.index("Source"); i_ex = h.index("Instructions Executed")
tot = sum(int(x[i_s] or 0) for x in data)
if len(sys.argv) > 2:
    cnt = sys.argv[2]
else:
    w = collections.Counter()
    for x in data:
        w[x[i_ex]] += int(x[i_s] or 0)
    cnt = w.most_common(1)[0][0]
idx = [k for k, x in enumerate(data) if x[i_ex] == cnt]
ssum = 0
for k in range(idx[0] - 2, idx[-1] + 3):
    x = data[k]
    s = int(x[i_s] or 0)
    ssum += s
    print(f"{k:5d} {s:6d} {x[i_ex]:>8s} {x[i_src][:100]}")
print("body instructions", len(idx), "samples", ssum, "of", tot)
