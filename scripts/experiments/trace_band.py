"""Per-band trace of the round-2 band kernel (-DNW_TRACE=1 build, bench.py --trace):
python scripts/trace_band.py trace.npy n [ghz]"""
import sys
import numpy as np
t = np.load(sys.argv[1]).astype(np.float64); n = int(sys.argv[2]); ghz = float(sys.argv[3]) if len(sys.argv) > 3 else 1.965
t = t[t[:, 1] > 0]
t = t[np.argsort(t[:, 0])]
t0 = t[:, 1].min()
steps = n + 31
print(f"bands={len(t)} span={(t[:, 2].max() - t0) / 1e3:.1f} us")
names = ["ready", "outring", "border", "events", "steady"]
for k in sorted(set([0, 1, 2, 3, 4, 5, len(t) // 2, len(t) // 2 + 1, len(t) - 2, len(t) - 1])):
    if k >= len(t):
        continue
    dur = (t[k, 2] - t[k, 1]) / 1e3
    cyc = dur * 1e3 * ghz
    ph = [t[k, 4], t[k, 5], t[k, 6], t[k, 7], t[k, 8]]
    nsteady = max(1.0, (n // 16 - 2))
    print(f"band {int(t[k,0]):4d} sm {int(t[k,3]):3d} start {(t[k,1]-t0)/1e3:8.1f} us dur {dur:8.1f} us = {cyc/steps:6.1f} cyc/step | "
          + " ".join(f"{nm} {v/steps:6.1f}" for nm, v in zip(names, ph)) + f" | steady/step {t[k,8]/(16*nsteady):6.1f}")
st = (t[:, 9] - t0) / 1e3
run = (t[:, 2] - t[:, 9]) / 1e3
print("first border valid (us): band 0 %.1f, 1 %.1f, 2 %.1f, 64 %.1f, 128 %.1f, last %.1f" % (st[0], st[1], st[2], st[min(64, len(st)-1)], st[min(128, len(st)-1)], st[-1]))
print("run after first border (us): band 0 %.1f, 1 %.1f, 128 %.1f, last %.1f -> cyc/step %.1f %.1f %.1f %.1f" % (
    run[0], run[1], run[min(128, len(run)-1)], run[-1], *(x * 1e3 * ghz / steps for x in (run[0], run[1], run[min(128, len(run)-1)], run[-1]))))
hop = np.diff(st)
print("hop (first-border) us: even->odd median %.2f, odd->even median %.2f" % (np.median(hop[0::2]), np.median(hop[1::2])))

