"""Band-to-band handoff latency from bench.py --trace (the *_hops.npy file): for consumer band k
and border block q, the producer (band k-1) wrote the block's last row at its step 16q+46
(event q+2, 14/16 into the block); the consumer recorded when it found the block valid."""
import sys
import numpy as np
h = np.load(sys.argv[1]).astype(np.float64)  # [band][0: event start, 1: block valid][q]
nb = h.shape[0]
for k in range(1, min(nb, 8)):
    T = h[k - 1, 0]
    D = h[k, 1]
    q = np.arange(100, 1900)
    pub = T[q + 2] + 14 / 16 * (T[q + 3] - T[q + 2])
    lat = D[q] - pub
    start_lag = h[k, 0][q] - h[k - 1, 0][q]
    print(f"band {k}: handoff latency median {np.median(lat):8.0f} ns  p10 {np.percentile(lat, 10):8.0f}  p90 {np.percentile(lat, 90):8.0f};"
          f"  event-start lag vs band {k-1}: median {np.median(start_lag):8.0f} ns; block period {np.median(np.diff(T[q])):6.0f} ns")
