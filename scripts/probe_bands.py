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


if __name__ == "__main__" and not (len(sys.argv) > 3 and sys.argv[3] == "global"):
    main()


def global_source_probe(n=32768, tile=128, epoch=5):
    """One band whose left border comes from an already-published (valid) global halo."""
    W = nwb.nw_band_width(tile)
    S, R = inputs.device_problem(n, 10, device="cuda")
    S1, R1 = S[:, : W + 1], R[:, : W + 1]
    vals = S[:, 0].to(torch.int64) & 0xFFFFFFFF
    halo = torch.zeros(n + 2, dtype=torch.int64, device="cuda")
    halo[: n + 1] = (epoch << 32) | vals
    for label, kw in (("plain", {}), ("global halo", {"halo_in": halo, "epoch": epoch})):
        for _ in range(2):
            nwb.nw_fill_sharded(S1, R1, 10, tile=tile, **kw)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(3):
            nwb.nw_fill_sharded(S1, R1, 10, tile=tile, **kw)
        e1.record()
        torch.cuda.synchronize()
        print(f"1 band, {label:12s}: {e0.elapsed_time(e1) / 3:.3f} ms", flush=True)


if __name__ == "__main__" and len(sys.argv) > 3 and sys.argv[3] == "global":
    global_source_probe(int(sys.argv[1]), int(sys.argv[2]))
