"""Warp-stall samples per CUDA source line (inlined lines attributed to their own line) from an
ncu report captured with -lineinfo and --import-source:  python scripts/ncu_lines.py rep [top]"""
import csv, io, subprocess, sys, collections
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
rows = list(csv.reader(io.StringIO(out)))
cur_file, h = None, None
agg = collections.defaultdict(lambda: [0, 0, collections.Counter(), ""])
tot = 0
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        cur_file = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        h = r
        continue
    if h is None or len(r) < 8:
        continue
    if r[0]:  # a source line row (aggregate of its SASS)
        ln = (cur_file, int(r[0]))
        num = lambda x: int(x) if x.isdigit() else 0
        s = num(r[4])
        a = agg[ln]
        a[0] += s
        a[1] += num(r[7])
        a[3] = r[1][:90]
        for i, name in enumerate(h):
            if name.startswith("stall_") and "Not Issued" not in name and i < len(r) and r[i].isdigit():
                a[2][name[6:]] += int(r[i])
        tot += s
print("total samples", tot)
for (f, ln), (s, ex, st, src) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    reasons = ",".join(f"{k}:{v}" for k, v in st.most_common(3))
    print(f"{f}:{ln:5d} {s:7d} {100*s/max(tot,1):5.1f}% ex={ex:>9d} [{reasons}] {src}")
