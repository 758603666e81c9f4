#!/usr/bin/env python
"""Decompose the persistent kernel's time: n rows x w columns for growing w (1, 2, 4, ... bands).

T(w) ~ n * t_row + (bands - 1) * lag; a 1-band strip gives the per-row cost of one warp, the
slope over bands gives the band-to-band lag.  Uses nw_fill_sharded on a local (n+1) x (w+1)
strip with a plain left border (no halo).
"""
import json
import sys

import torch

sys.path.insert(0, ".")
import inputs  # noqa: E402
import paper_conf_sc_munksgaardhso22_b200 as nwb  # noqa: E402


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
    tile = int(sys.argv[2]) if len(sys.argv) > 2 else 128
    W = nwb.nw_band_width(tile)
    S_full, R_full = inputs.device_problem(n, 10, device="cuda")
    res = []
    for nb in (1, 2, 3, 4, 8, 16, 64, 256):
        w = min(nb * W, n)
        S = S_full[:, : w + 1]
        R = R_full[:, : w + 1]
        for _ in range(2):
            nwb.nw_fill_sharded(S, R, 10, tile=tile)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        reps = 3
        for _ in range(reps):
            nwb.nw_fill_sharded(S, R, 10, tile=tile)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / reps
        res.append((nb, w, ms))
        print(f"bands {nb:4d}  w {w:6d}  {ms:8.3f} ms  per-row {ms * 1e6 / n:7.1f} ns  "
              f"GCUPS {n * w / ms / 1e6:8.1f}", flush=True)
    print(json.dumps(res))


if __name__ == "__main__":
    main()
