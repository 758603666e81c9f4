#!/usr/bin/env python
"""Summarise a per-band trace written by `bench.py --trace` (nw_debug_set_trace).

Each row: {task, start_ns, end_ns, smid}.  Prints the launch span, per-band sweep time, the
band-to-band start lag (the wavefront ramp), and how many bands were in flight over time.
"""
import sys

import numpy as np


def main(path, n=None):
    t = np.load(path).astype(np.int64)
    t = t[t[:, 2] > 0].astype(np.int64)
    t = t[np.argsort(t[:, 0])]
    t0 = t[:, 1].min()
    st, en = (t[:, 1] - t0) / 1e3, (t[:, 2] - t0) / 1e3   # us
    dur = en - st
    lag = np.diff(st)
    span = en.max()
    print(f"bands={len(t)}  span={span:.1f} us  sweep mean={dur.mean():.1f} us (min {dur.min():.1f}, "
          f"max {dur.max():.1f})")
    print(f"start lag band->band: mean={lag.mean():.2f} us median={np.median(lag):.2f} us "
          f"p90={np.percentile(lag, 90):.2f} us; last band starts at {st.max():.1f} us")
    if n:
        print(f"  per-row step time (sweep/n) = {dur.mean() / n * 1e3:.1f} ns; lag in steps ~ "
              f"{np.median(lag) / (dur.mean() / n):.1f}")
    grid = np.linspace(0, span, 21)
    act = [int(((st <= g) & (en > g)).sum()) for g in grid]
    print("bands in flight over the launch:", act)
    blk = t[:, 3] >> 16
    t[:, 3] &= 0xFFFF
    print("distinct SMs:", len(np.unique(t[:, 3])))
    if n and blk.max() > 0:
        print(f"  steady-state step blocks: mean {blk.mean() / n:.1f} cycles/row, band0 {blk[0] / n:.1f}")
    if t.shape[1] >= 8:
        tot = t[:, 7].astype(float)
        cols = [("events", 4), ("ref waits", 5), ("border spins", 6)]
        if t.shape[1] >= 10:
            cols += [("staging busy", 8), ("staging wait", 9)]
        for name, col in cols:
            fr = t[:, col] / np.maximum(tot, 1)
            print(f"  {name:13s}: mean {fr.mean()*100:5.1f}% of task cycles (band0 {fr[0]*100:5.1f}%)")
        if n:
            comp = (tot - t[:, 4]) / n
            print(f"  step cycles/row excluding events+spins: mean {comp.mean():.1f}, band0 {comp[0]:.1f};"
                  f" total cycles/row band0 {tot[0]/n:.1f}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else None)
