#!/usr/bin/env python3
"""Deterministic drivers for ncu captures of the benched configuration (run them under
`ncu --replay-mode application ...`: application replay re-runs this process per metric pass
instead of saving / restoring device and pinned-host memory, which is what got kernel-replay
captures of the 57 GB pinned host tier OOM-killed in round 1).

  --what traffic : the bench.py workload (host tier on by default), W warm-up + K timed
                   extracts of distinct batches, 256 MiB L2 flush before each -- the per-launch
                   DRAM / PCIe bytes of the dominant kernel (profiles/traffic.json).
  --what calibrate : ugache_calibrate (A0) through the ctx of this workload.
  --what fig13   : Fig. 13 analog: the locally hit keys of one batch removed,
                   the remaining host keys extracted by the factored kernel and by random
                   dispatch (same placement), one warm-up + one measured launch each, L2
                   flushed before each.  Without ncu it also prints CUDA-event times and the
                   achieved host-link GB/s of both.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--what", default="traffic", choices=["traffic", "fig13", "calibrate"])
    ap.add_argument("--workload", default="gnn_pa")
    ap.add_argument("--cache-ratio", type=float, default=None)
    ap.add_argument("--no-host-tier", dest="host_tier", action="store_false", default=True)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--reps", type=int, default=5, help="fig13: timed repetitions without ncu")
    args = ap.parse_args()
    import torch
    import synth
    from paper_conf_sosp_songz0c23_b200 import UGache, make_config, solve
    wl = synth.get_workload(args.workload)
    if args.cache_ratio is not None:
        from dataclasses import replace
        wl = replace(wl, cache_ratio=args.cache_ratio)
    torch.cuda.set_device(0)
    table = synth.HostTable(wl.num_rows, wl.row_bytes)
    table.fill()
    h = synth.hotness(wl)
    cfg = make_config(wl.num_rows, wl.row_bytes, wl.capacity_rows, host_tier=args.host_tier)
    plan, order = solve(cfg, h)
    del h
    cache = UGache(table, wl.num_rows, wl.row_bytes, wl.capacity_rows, plan=plan, order=order,
                   host_tier=args.host_tier)
    cache.fill()
    torch.cuda.synchronize()
    R = wl.row_bytes
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    nb = args.warmup + args.steps
    batches = [torch.from_numpy(synth.make_batch(wl, 0, i)).cuda() for i in range(max(nb, 1))]
    out = torch.empty((batches[0].numel(), R), dtype=torch.uint8, device="cuda")

    def run(keys, o):
        flush.fill_(1)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        cache.extract(keys, o)
        e.record()
        torch.cuda.synchronize()
        return s.elapsed_time(e)

    res = {"what": args.what, "workload": wl.name, "cache_ratio": wl.cache_ratio, "host_tier": args.host_tier}
    if args.what == "calibrate":
        res["calibration"] = cache.calibrate()
    elif args.what == "traffic":
        ms = [run(batches[i], out) for i in range(nb)]
        per, _ = cache.last_batch_stats()
        res.update(ms=ms[args.warmup:], path=cache.last_extract_path(), per_source=per.tolist())
    else:
        loc, _ = cache.export_placement()
        b0 = batches[0].cpu().numpy()
        hk = b0[(loc[b0] >> np.uint64(56)) == np.uint64(1)]
        del loc
        dk = torch.from_numpy(np.ascontiguousarray(hk)).cuda()
        ho = torch.empty((len(hk), R), dtype=torch.uint8, device="cuda")
        cache.set_stream("off")                                 # the two-phase factored kernel
        for mode in ("factored", "random"):
            cache.set_mode(mode)
            run(dk, ho)                                         # warm-up (the skipped launch)
            t = [run(dk, ho) for _ in range(args.reps)]
            res[mode] = {"ms": statistics.median(t), "host_keys": int(len(hk)),
                         "host_gbs": len(hk) * R / (statistics.median(t) * 1e-3) / 1e9,
                         "path": cache.last_extract_path()}
    print(json.dumps(res), flush=True)
    cache.close()
    table.close()


if __name__ == "__main__":
    main()
