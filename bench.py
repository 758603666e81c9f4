#!/usr/bin/env python
"""bench.py — NW GCUPS + HBM roofline of the B200 wavefront (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C] [--tile B] [--impl ours|reference]

One step = one pass of the whole hot path (one nw_fill / nw_fill_batch call = ONE kernel launch)
over the config's synthetic input, resident in HBM.  Defaults: N=1 -> config 3 (n=32768, the
headline, BASELINE.json configs[2]); N>1 (torchrun) -> config 4 (4096 independent n=2048 pairs
split contiguously over the ranks, no collective on the data path).  Prints ONE JSON line on
rank 0.  Inputs (8.6 GB at config 3) are far larger than the 126 MB L2, so no flush is needed.

--impl reference times the CPU oracle (oracle/nw_ref.c, single-threaded) on a bounded sample of
the same workload on the host cores (rank 0 only), as the driver's reference arm.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIGS = {
    1: dict(workload="nw_n1024_p10_tile16", n=1024, batch=1, tile=16),
    2: dict(workload="nw_n16384_p10", n=16384, batch=1, tile=64),
    3: dict(workload="nw_n32768_p10", n=32768, batch=1, tile=0),
    4: dict(workload="nw_batch4096_n2048_p10", n=2048, batch=4096, tile=0),
    5: dict(workload="nw_n65536_p10_strips", n=65536, batch=1, tile=0, strips=True),
}
PENALTY = 10
METRIC = "NW GCUPS (interior cell updates / s), bit-exact vs CPU oracle"


def env_int(k, d):
    try:
        return int(os.environ.get(k, d))
    except ValueError:
        return d


class Clocks:
    """nvidia-smi sampler during the timed region (clocks + throttle reasons)."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index, self.rows, self._stop = index, [], threading.Event()
        self._t = threading.Thread(target=self._run, daemon=True)

    def _run(self):
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True,
                                     timeout=5).stdout.strip()
                if out:
                    self.rows.append([x.strip() for x in out.split(",")])
            except Exception:
                pass
            self._stop.wait(0.2)

    def __enter__(self):
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        self._t.join(timeout=10)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if len(r) > 4 + i and r[4 + i] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            j = json.load(f)
        return float(j["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, burst copy)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def ncu_traffic(workload, tile):
    """DRAM bytes per launch of the dominant kernel from the committed ncu --set full summary."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            j = json.load(f)
        return j.get(f"{workload}/tile{tile}")
    except Exception:
        return None


# Cycles of one wavefront step of one band in isolation (a warp per SM sub-partition, no staging
# stalls), measured on B200 with scripts/ubench_mw.cu (round 2): K = 8: 88.1; K = 4 one band per
# SM: 53.1; K = 4 two bands per SM: 52.2 (each).
STEP_CYCLES = {8: 88.1, 4: 53.1}


def latency_floor(n, B, tile, nwb, kern_ms, clocks, variant, world, strips):
    """The other roofline of the wavefront: its critical path.  A band's warp needs n + 31 steps
    (its 32 lanes are skewed by one row) and band k+1 can start no earlier than 32 steps after band
    k, so one pair takes at least n + 31 * nbands steps; in pair mode (large batches) a CTA sweeps
    its pairs' bands back to back: ceil(pairs / CTAs) * nbands * (n + 31) steps.  frac = that floor
    at the isolated step time / the measured kernel time."""
    if variant not in ("strip", "seq") or strips:
        return None
    W = nwb.nw_band_width(tile)
    K = W // 32
    nb = -(-n // W)
    c = STEP_CYCLES[K]
    mhz = clocks.get("sm_mhz") or 1965.0
    if B == 1:
        steps = n + 31 * nb
        how = f"n + 31 * nbands = {n} + 31 * {nb}"
    else:
        ki = nwb.nw_kernel_info(tile)
        grid = ki["ctas_per_sm"] * ki["num_sms"]
        per = -(-(B // world) // grid)
        steps = per * nb * (n + 31)
        how = f"ceil(pairs / {grid} CTAs) * nbands * (n + 31) = {per} * {nb} * {n + 31}"
    floor_ms = steps * c / (mhz * 1e3)
    return {"bound": "wavefront critical path", "critical_steps": steps, "steps_formula": how,
            "step_cycles_isolated": c, "step_cycles_source": "scripts/ubench_mw.cu (B200, round 2)",
            "sm_mhz": mhz, "floor_ms": floor_ms, "frac": floor_ms / kern_ms,
            "cycles_per_critical_step": kern_ms * mhz * 1e3 / steps}


def cpu_baseline(cfg, gpu_score=None):
    """The oracle as it stands (single-threaded C) on a bounded sample of the workload; when the
    GPU's result is given (device tensor), every oracle row / pair is compared with it (outside the
    oracle's timing)."""
    import numpy as np

    import inputs
    import oracle
    n, p = cfg["n"], PENALTY
    if cfg["batch"] == 1:
        # whole matrix, streamed (O(n) memory): rows generated block by block from the same seed
        a, b = inputs.gen_pair(n, inputs.SEED)
        row0 = -np.arange(n + 1, dtype=np.int32) * p
        st = oracle.NwRefStream(n, p, row0)
        t_or = 0.0
        rows_done = 0
        budget = float(os.environ.get("NW_CPU_BASELINE_S", "25"))
        exact = None if gpu_score is None else True
        for i0 in range(1, n + 1, 1024):
            i1 = min(n + 1, i0 + 1024)
            blk = inputs.build_ref_block(a, b, i0, i1)
            col0 = (-np.arange(i0, i1, dtype=np.int64) * p).astype(np.int32)
            t = time.perf_counter()
            out = st.rows(blk, col0, want_out=True)  # (the oracle produces the rows; timed either way)
            t_or += time.perf_counter() - t
            rows_done = i1 - 1
            if gpu_score is not None:
                exact = exact and bool(np.array_equal(out, gpu_score[i0:i1, : n + 1].cpu().numpy()))
            if t_or > budget:
                break
        st.close()
        cells = rows_done * n
        sample = f"rows 1..{rows_done} of the n={n} matrix (streaming oracle, {cells:.3e} cells)"
        return {"value": cells / t_or / 1e9, "unit": "GCUPS", "cores": 1, "kind": "oracle",
                "sample": sample, "seconds": t_or, "bit_exact_rows": rows_done if exact else None,
                "bit_exact": exact}
    # batch: the first pairs of the batch, one by one
    t_or, cells, k = 0.0, 0, 0
    exact = None if gpu_score is None else True
    budget = float(os.environ.get("NW_CPU_BASELINE_S", "15"))
    while t_or < budget and k < cfg["batch"]:
        s, r = inputs.make_problem(n, p, seed=inputs.pair_seed(k))
        t = time.perf_counter()
        want = oracle.nw_ref(s, r, p)
        t_or += time.perf_counter() - t
        if gpu_score is not None:
            exact = exact and bool(np.array_equal(want, gpu_score[k].cpu().numpy()))
        cells += n * n
        k += 1
    return {"value": cells / t_or / 1e9, "unit": "GCUPS", "cores": 1, "kind": "oracle",
            "sample": f"first {k} of {cfg['batch']} pairs (n={n})", "seconds": t_or,
            "bit_exact_pairs": k if exact else None, "bit_exact": exact}


def run_reference(args, cfg, rank):
    if rank != 0:
        return
    import oracle
    oracle.build()
    steps = []
    # each step is a bounded sample so the whole --steps K --warmup W run stays within minutes
    os.environ["NW_CPU_BASELINE_S"] = str(min(25.0, 150.0 / (args.warmup + args.steps)))
    for _ in range(args.warmup + args.steps):
        steps.append(cpu_baseline(dict(cfg), None))
    timed = steps[args.warmup:]
    v = statistics.mean(s["value"] for s in timed)
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "GCUPS", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "higher_is_better": True, "dtype": "int32",
            "data": "synthetic", "config": {"workload": cfg["workload"], "n": cfg["n"], "batch": cfg["batch"],
                                            "penalty": PENALTY},
            "cpu_baseline": {"value": v, "unit": "GCUPS", "cores": 1, "kind": "oracle",
                             "sample": timed[0]["sample"]},
            "e2e": {"value": v, "unit": "GCUPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=0)
    ap.add_argument("--tile", type=int, default=-1)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--layout", default="rodinia", choices=["rodinia", "aligned"],
                    help="device matrix layout: the Rodinia pitch n+1 (default) or 16-byte aligned interior "
                         "rows (pitch rounded up to 4 elements; 16-byte staging copies)")
    ap.add_argument("--cluster", action="store_true",
                    help="experiment: one pair as thread-block clusters handing the border over through DSMEM")
    ap.add_argument("--trace", default="", help="write per-band {task,start,end,smid} of one extra launch here (.npy)")
    ap.add_argument("--variant", default="strip", choices=["strip", "diagonal", "unopt", "seq"],
                    help="ablation: the paper's per-diagonal structure (Opt) / Unopt instead of the "
                         "persistent kernel")
    args = ap.parse_args()
    world = env_int("WORLD_SIZE", 1)
    rank = env_int("RANK", 0)
    local_rank = env_int("LOCAL_RANK", 0)
    cfg_id = args.config or (3 if world == 1 else 4)
    cfg = dict(CONFIGS[cfg_id])
    if args.tile >= 0:
        cfg["tile"] = args.tile
    args.warmup = max(args.warmup, 3)
    if args.impl == "reference":
        return run_reference(args, cfg, rank)

    import numpy as np
    import torch

    import inputs
    import paper_conf_sc_munksgaardhso22_b200 as nwb
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if args.cluster:
        nwb.nw_debug_set_cluster(True)
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=dev)
    n, p, tile = cfg["n"], PENALTY, cfg["tile"]
    B = cfg["batch"]
    strips = cfg.get("strips", False) and world > 1
    if strips:
        # config 5: column strips of one n=65536 pair, right border pushed to the next rank over
        # NVLink from inside the kernel (torch symmetric memory peer pointers), one barrier per call
        from paper_conf_sc_munksgaardhso22_b200 import dist as nwdist
        shard = nwdist.StripShard(n, p, inputs.SEED, tile=tile)
        S = shard.score

        def step():
            shard.fill()
            shard.barrier()
        cells_local = n * shard.strip.w
    elif B > 1:
        from paper_conf_sc_munksgaardhso22_b200 import dist as nwdist
        lo, hi = nwdist.pair_range(B, world, rank)
        nb = hi - lo
        if args.layout == "aligned":
            S, R = inputs.device_aligned_batch(nb, n, dev), inputs.device_aligned_batch(nb, n, dev)
        else:
            S = torch.empty((nb, n + 1, n + 1), dtype=torch.int32, device=dev)
            R = torch.empty((nb, n + 1, n + 1), dtype=torch.int32, device=dev)
        for k in range(nb):
            inputs.device_problem(n, p, seed=inputs.pair_seed(lo + k), device=dev, score=S[k], ref=R[k])

        def step():
            nwb.nw_fill_batch(S, R, p, tile)
        cells_local = nb * n * n
    else:
        S, R = inputs.device_problem(n, p, device=dev, layout=args.layout)
        if args.variant == "seq":       # NEXT-2: ref generated on chip from the sequences
            a_h, b_h = inputs.gen_pair(n, inputs.SEED)
            Ad, Bd = torch.from_numpy(a_h).to(dev), torch.from_numpy(b_h).to(dev)
            tab = inputs.blosum62()
            del R
            R = None

            def step():
                nwb.nw_fill_seq(S, Ad, Bd, tab, p, tile)
        elif args.variant == "strip":
            def step():
                nwb.nw_fill(S, R, p, tile)
        else:
            if tile not in (16, 32, 64):
                tile = cfg["tile"] = 16
            fn = nwb.nw_fill_diagonal if args.variant == "diagonal" else nwb.nw_fill_unopt

            def step():
                fn(S, R, p, tile)
        cells_local = n * n
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream()
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    with Clocks(local_rank) as clk:
        time.sleep(0.3)
        torch.cuda.synchronize()
        t0 = torch.cuda.Event(enable_timing=True)
        t1 = torch.cuda.Event(enable_timing=True)
        t0.record(stream)
        for e0, e1 in ev:
            e0.record(stream)
            step()
            e1.record(stream)
        t1.record(stream)
        torch.cuda.synchronize()
    total_ms = t0.elapsed_time(t1)
    per_launch = [e0.elapsed_time(e1) for e0, e1 in ev]
    if world > 1:
        tt = torch.tensor([total_ms], device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        total_ms = float(tt.item())
    cells_total = cells_local if world == 1 else B * n * n   # (strips: B = 1, all n*n cells)
    ms_per_step = total_ms / args.steps
    value = cells_total / (ms_per_step * 1e-3) / 1e9
    # roofline of the (only) kernel: 8 algorithmic bytes per interior cell (ref read + score write)
    kern_ms = statistics.mean(per_launch)   # == the step: one launch per step for the strip kernel
    bpc = 4.0 if args.variant == "seq" else 8.0   # algorithmic HBM bytes per cell
    achieved = bpc * cells_local / (kern_ms * 1e-3) / 1e9
    peak, peak_src = measured_peaks()
    roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
            "traffic": ncu_traffic(cfg["workload"], tile),
            "traffic_source": "profiles/ncu_traffic.json: dram__bytes_read.sum + dram__bytes_write.sum per launch "
                              "from the latest ncu --set full capture of this kernel (profiles/r02c_*)",
            "peak_source": peak_src,
            "algorithmic_bytes_per_launch": int(bpc * cells_local),
            "kernel": ("nw_wave_kernel<WaveCfg<K=%d, SEQ=%d>> (W = %d columns per band)"
                       % (nwb.nw_band_width(tile) // 32, int(args.variant == "seq"), nwb.nw_band_width(tile)))
            if args.variant in ("strip", "seq")
            else f"nw_diag_kernel<{tile}> x{nwb.nw_launch_count(1, n, tile)} launches (+copies: unopt)",
            "kernel_ms_mean": kern_ms, "kernel_ms_median": statistics.median(per_launch)}
    roof["latency"] = latency_floor(n, B if not strips else 1, tile, nwb, kern_ms, clk.summary(), args.variant,
                                    world, strips)
    out = {"metric": METRIC, "value": value, "unit": "GCUPS", "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
           "scaling": "strong" if world > 1 else "weak", "vs_baseline": None, "dtype": "int32",
           "data": "synthetic (splitmix64 seq 7, BLOSUM62 ref, global-alignment borders)",
           "config": {"workload": cfg["workload"], "n": n, "batch": B, "penalty": p, "tile": tile,
                      "band_width": nwb.nw_band_width(tile), "pairs_per_rank": B // world if B > 1 else 1,
                      "l2": "inputs %.1f GB >> 126 MB L2 (no flush needed)" % (8.0 * (n + 1) ** 2 * B / 1e9),
                      "layout": "strips (pitch w+1)" if strips else (
                          "aligned: interior rows 16-byte aligned, pitch %d" % ((n + 4) & ~3) if args.layout == "aligned"
                          else "rodinia: pitch n+1"),
                      "parallelism": (f"strips{world}" if strips else f"dp{world}") if world > 1 else "single"},
           "roofline": roof,
           "gpu_launches": args.steps * nwb.nw_launch_count({"strip": 0, "seq": 0, "diagonal": 1, "unopt": 2}[args.variant], n, tile),
           "variant": args.variant,
           "clocks": clk.summary()}
    # ---- NEXT-3: traceback of the filled matrix (outside the timed fill; reported beside it)
    if not strips and args.variant in ("strip", "seq") and R is not None:
        SB, RB = (S, R) if B > 1 else (S.unsqueeze(0), R.unsqueeze(0))
        tb_ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(4)]
        for e0, e1 in tb_ev:
            e0.record(stream)
            ops, length = nwb.nw_traceback_batch(SB, RB, p)
            e1.record(stream)
        torch.cuda.synchronize()
        tb_ms = statistics.median([e0.elapsed_time(e1) for e0, e1 in tb_ev[1:]])
        steps_total = int(length.to(torch.int64).sum().item())
        out["traceback"] = {"ms": tb_ms, "pairs": int(SB.shape[0]), "path_steps": steps_total,
                            "msteps_per_s": steps_total / (tb_ms * 1e-3) / 1e6, "launches": 2,
                            "bound": "latency (one dependent walk per pair, 33x33 windows)"}
    if args.trace and not strips:
        ntask = (B if B > 1 else 1) * -(-n // nwb.nw_band_width(tile))
        tbuf = torch.zeros(16 * ntask, dtype=torch.int64, device=dev)
        tb = tbuf[: 8 * ntask].view(ntask, 8)
        nwb.nw_debug_set_trace(tb)
        step()
        torch.cuda.synchronize()
        nwb.nw_debug_set_trace(None)
        tt = tbuf.cpu().numpy()
        np.save(args.trace, np.concatenate([tt[: 8 * ntask].reshape(ntask, 8), tt[8 * ntask:].reshape(ntask, 8)], 1))
    # ---- e2e through the public C ABI with host buffers (H2D + kernel + D2H inside the timing)
    if B == 1 and args.e2e_steps > 0 and args.variant == "strip" and not strips:
        hs = torch.empty((n + 1, n + 1), dtype=torch.int32, pin_memory=True)
        hr = torch.empty((n + 1, n + 1), dtype=torch.int32, pin_memory=True)
        hr.copy_(R.cpu())
        hs[0].copy_(S[0].cpu())
        hs[:, 0].copy_(S[:, 0].cpu())
        hs_np, hr_np = hs.numpy(), hr.numpy()
        nwb.nw_fill_host(hs_np, hr_np, p, tile, local_rank)       # warm-up (allocations)
        t = time.perf_counter()
        for _ in range(args.e2e_steps):
            nwb.nw_fill_host(hs_np, hr_np, p, tile, local_rank)
        e2e_s = (time.perf_counter() - t) / args.e2e_steps
        out["e2e"] = {"value": cells_local / e2e_s / 1e9, "unit": "GCUPS",
                      "h2d_bytes_per_step": 4 * (n + 1) ** 2 + 4 * (2 * n + 1),
                      "d2h_bytes_per_step": 4 * (n + 1) ** 2, "ms_per_step": e2e_s * 1e3,
                      "api": "nw_fill_host (pinned host buffers)"}
        out["gpu_launches_e2e"] = args.e2e_steps + 1
        nwb.nw_release_workspace()
        del hs, hr
    elif B > 1 and args.e2e_steps > 0:
        # batch: end to end through the public host API (nw_fill_batch_host) on a bounded
        # sub-batch per rank, pinned host buffers (the kernel reads ref and writes score over the
        # host link itself: zero copy)
        sb = min(nb, 32)
        hr = torch.empty((sb, n + 1, n + 1), dtype=torch.int32, pin_memory=True)
        hs = torch.empty((sb, n + 1, n + 1), dtype=torch.int32, pin_memory=True)
        hr.copy_(R[:sb].cpu())
        hs.copy_(S[:sb].cpu())
        hs_np, hr_np = hs.numpy(), hr.numpy()
        nwb.nw_fill_batch_host(hs_np, hr_np, p, tile, local_rank)
        if world > 1:
            dist.barrier()
        t = time.perf_counter()
        for _ in range(args.e2e_steps):
            nwb.nw_fill_batch_host(hs_np, hr_np, p, tile, local_rank)
        e2e_s = (time.perf_counter() - t) / args.e2e_steps
        if world > 1:
            tt = torch.tensor([e2e_s], device=dev)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            e2e_s = float(tt.item())
        out["e2e"] = {"value": world * sb * n * n / e2e_s / 1e9, "unit": "GCUPS",
                      "h2d_bytes_per_step": world * sb * (4 * (n + 1) ** 2 + 4 * (2 * n + 1)),
                      "d2h_bytes_per_step": world * 4 * sb * (n + 1) ** 2, "ms_per_step": e2e_s * 1e3,
                      "api": f"nw_fill_batch_host on a {sb}-pair sub-batch per rank (pinned host buffers)"}
        out["gpu_launches_e2e"] = args.e2e_steps + 1
        nwb.nw_release_workspace()
        del hr, hs
    if rank == 0 and not args.no_cpu:
        # (strips: the local strip is not the whole matrix; batch: this rank's first pairs are the
        # global pairs lo.. -- rank 0 holds the first)
        out["cpu_baseline"] = cpu_baseline(cfg, S if not strips else None)
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
