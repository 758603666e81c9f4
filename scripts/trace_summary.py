"""One-line summary of a wave-kernel trace: band-0 cycles/row split, mean spins, span."""
import sys
import numpy as np
t = np.load(sys.argv[1]).astype(np.int64)
n = int(sys.argv[2]) if len(sys.argv) > 2 else 32768
t = t[t[:, 2] > 0]
ghz = 1.965
tot = (t[:, 2] - t[:, 1]) * ghz
span = (t[:, 2].max() - t[:, 1].min()) / 1e3
print(f"bands={len(t)} span={span:.0f}us band0: {tot[0]/n:.1f} cyc/row (events {t[0,4]/n:.1f}, cp-wait {t[0,7]/n:.1f}, spin {t[0,6]/n:.1f}); "
      f"mean: total {tot.mean()/n:.1f} events {(t[:,4]/n).mean():.1f} spin {(t[:,6]/n).mean():.1f} bp {(t[:,5]/n).mean():.1f}; "
      f"last band ends {(t[-1,2]-t[:,1].min())/1e3:.0f}us, band0 ends {(t[0,2]-t[:,1].min())/1e3:.0f}us")
if t.shape[1] >= 12:
    ph = t[:, 8:12] / n
    print("event phases cyc/row (publish, staging wait, cp.async+sync, border+bp): band0", np.round(ph[0], 1).tolist(), "mean", np.round(ph.mean(0), 1).tolist())
