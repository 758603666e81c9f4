"""Per-chunk timing of band 0 / 1 (trace build, bench.py --trace: *_chunks.npy): for block Q, when
ready(Q) was observed vs when its ref row chunk Q+1 copy was issued and its score chunk Q-NSB stored.
python scripts/trace_chunks.py file_chunks.npy nsb"""
import sys
import numpy as np
c = np.load(sys.argv[1]).astype(np.float64); nsb = int(sys.argv[2]) if len(sys.argv) > 2 else 6
for b in (0, 1):
    st0, st1, cp, rd = c[4 * b], c[4 * b + 1], c[4 * b + 2], c[4 * b + 3]
    Q = np.arange(100, 1900)
    print(f"band {b}: block period {np.median(np.diff(rd[Q])):.0f} ns")
    print(f"   ready(Q) - copy issue of row chunk Q+1: median {np.median(rd[Q] - cp[Q + 1]):.0f} ns  p10 {np.percentile(rd[Q] - cp[Q + 1], 10):.0f}  p90 {np.percentile(rd[Q] - cp[Q + 1], 90):.0f}")
    print(f"   ready(Q) - store done of chunk Q-{nsb}: median {np.median(rd[Q] - st1[Q - nsb]):.0f} ns")
    print(f"   store duration: median {np.median(st1[Q] - st0[Q]):.0f} ns; copy issue lead over its need (ready(k-1) - issue(k)) see above")
    print(f"   copy issue(k) - ready(k-5) (when the slot became free: cdone(k-5) arrives at event k-4): median {np.median(cp[Q + 1] - rd[Q - 4]):.0f} ns")
