"""Print the SASS of an ncu report in address order with per-instruction stall samples,
restricted to instructions executed about `count` times (e.g. one loop body)."""
import csv, io, subprocess, sys
rep, lo, hi = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[1]; data = rows[2:]
ix = {k: h.index(k) for k in ["Source", "Instructions Executed", "Warp Stall Sampling (All Samples)", "stall_wait", "stall_short_sb", "stall_long_sb", "stall_branch_resolving", "stall_selected", "stall_dispatch", "stall_no_inst"]}
tot = 0
sel = [x for x in data if lo <= int(x[ix["Instructions Executed"]] or 0) <= hi]
agg = {k: 0 for k in ix if k.startswith("stall") or k.startswith("Warp")}
for x in sel:
    for k in agg: agg[k] += int(x[ix[k]] or 0)
print(len(sel), "instructions;", agg)
for x in sel:
    print(f"{x[0][-5:]} {x[ix['Warp Stall Sampling (All Samples)']]:>6s} w{x[ix['stall_wait']]:>5s} s{x[ix['stall_short_sb']]:>5s} l{x[ix['stall_long_sb']]:>5s} b{x[ix['stall_branch_resolving']]:>5s}  {x[ix['Source']][:90]}")
