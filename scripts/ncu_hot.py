"""Top SASS lines by warp-stall samples (with the dominant stall reasons) from an ncu report."""
import csv, io, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[1]
data = [x for x in rows[2:] if len(x) > 1 and (x[h.index("Warp Stall Sampling (All Samples)")] or "0").isdigit()]
i_s = h.index("Warp Stall Sampling (All Samples)"); i_src = h.index("Source"); i_ex = h.index("Instructions Executed")
stall_cols = [i for i, x in enumerate(h) if x.startswith("stall_") or "Stall" in x and i != i_s]
tot = sum(int(x[i_s] or 0) for x in data)
print("total samples", tot, "instructions", len(data))
for x in sorted(data, key=lambda x: -int(x[i_s] or 0))[:top]:
    print(f"{x[0][-5:]} {int(x[i_s]):7d} {100*int(x[i_s])/tot:5.1f}% ex={x[i_ex]:>10s}  {x[i_src][:80]}")
