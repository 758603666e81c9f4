"""Per-instruction stall breakdown of the compute warp's hottest loop (the steady 8-step sub-block):
python scripts/ncu_steady.py src.csv  (ncu -i rep --page source --csv --print-source sass > src.csv)"""
import collections, csv, io, sys
rows = list(csv.reader(open(sys.argv[1])))
while rows and "Address" not in rows[0]:
    rows = rows[1:]
h, data = rows[0], rows[1:]
ix = {k: h.index(k) for k in h}
i_s = ix["Warp Stall Sampling (All Samples)"]; i_ex = ix["Instructions Executed"]; i_src = ix["Source"]
stalls = [k for k in h if k.startswith("stall_") and "Not Issued" not in k]
w = collections.Counter()
for x in data:
    w[x[i_ex]] += int(x[i_s] or 0)
cnt = sys.argv[2] if len(sys.argv) > 2 else w.most_common(1)[0][0]
idx = [k for k, x in enumerate(data) if x[i_ex] == cnt]
tot = collections.Counter(); ssum = 0
for k in range(idx[0], idx[-1] + 1):
    x = data[k]
    s = int(x[i_s] or 0); ssum += s
    top = sorted(((int(float(x[ix[c]] or 0)), c[6:]) for c in stalls), reverse=True)[:3]
    for c in stalls: tot[c[6:]] += int(float(x[ix[c]] or 0))
    print(f"{s:6d} {x[i_ex]:>8s} {x[i_src][:70]:70s} " + " ".join(f"{c}:{v}" for v, c in top if v))
print("body instrs", idx[-1] - idx[0] + 1, "samples", ssum, "exec count", cnt)
print("stall totals:", ", ".join(f"{k}={v}" for k, v in tot.most_common(10)))
