"""Per-band trace summary (bench.py --trace): sweep time, per-step cycles, border spin and staging
wait of the compute warps:  python scripts/trace_quick.py trace.npy n [ghz]"""
import sys
import numpy as np
t = np.load(sys.argv[1]); n = int(sys.argv[2]); ghz = float(sys.argv[3]) if len(sys.argv) > 3 else 1.965
t = t[np.argsort(t[:, 0])]
t0 = t[:, 1].min()
dur = (t[:, 2] - t[:, 1]) / 1e3
spin = t[:, 6] / ghz / 1e3
wait = t[:, 7] / ghz / 1e3
bp = t[:, 5] / ghz / 1e3
steps = n + 31
sc = (t[:, 4] & ((1 << 44) - 1)).astype(np.float64)
sb = (t[:, 4] >> 44).astype(np.float64)
print(f"bands={len(t)} span={(t[:, 2].max() - t0) / 1e3:.1f} us; band0 sweep {dur[0]:.1f} us "
      f"({(dur[0] - wait[0]) * 1e3 * ghz / steps:.1f} cyc/step excl. staging waits)")
for k in sorted(set([0, 1, 2, len(t) // 2, len(t) - 1])):
    print(f"  band {k:4d}: start {(t[k, 1] - t0) / 1e3:8.1f} us sweep {dur[k]:8.1f} us spin {spin[k]:7.1f} us "
          f"staging-wait {wait[k]:7.1f} us bp {bp[k]:6.1f} us  cyc/step(excl spin+wait) {(dur[k] - spin[k] - wait[k]) * 1e3 * ghz / steps:6.1f}"
          f" steady-block cyc/step {sc[k] / max(sb[k], 1) / 16:6.1f} ({int(sb[k])} blocks)")
    if t.shape[1] >= 11:
        nev = (n + 31 + 15) // 16
        if t.shape[1] >= 14:
            nch = (n + 7) // 8
            print(f"      store warp: busy {t[k, 12] / nch:7.1f} cyc/chunk, gap before chunk {t[k, 13] / nch:7.1f} cyc/chunk")
        print(f"      per event cycles: publish+wait {t[k, 8] / nev:7.1f} (wait {t[k, 7] / nev:7.1f})  border {t[k, 9] / nev:7.1f} (spin {t[k, 6] / nev:7.1f})  bp+misc {t[k, 10] / nev:7.1f}  (wait on store warp only {t[k, 11] / nev:7.1f})  publish alone {t[k, 14] / nev:7.1f}")
