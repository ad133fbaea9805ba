#!/usr/bin/env python3
"""A0 calibration on one B200 (Fig. 6 analog): factored-gather time vs the
number of SMs dedicated to the host source, with and without host range ordering, on a
real workload placement.  Prints one JSON object per setting and a summary."""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="gnn_pa")
    ap.add_argument("--cache-ratio", type=float, default=None)
    ap.add_argument("--host-sms", default="1,2,4,6,8,12,16,24,32,48,64,96,128,140")
    ap.add_argument("--reps", type=int, default=6)
    ap.add_argument("--order", default="1,0")
    ap.add_argument("--random", action="store_true")
    ap.add_argument("--combos", default="", help="rows:warps,... (UGACHE_HOST_ROWS/WARPS per ctx)")
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
    cfg = make_config(wl.num_rows, wl.row_bytes, wl.capacity_rows)
    plan, order = solve(cfg, h)
    del h
    def new_cache():
        c = UGache(table, wl.num_rows, wl.row_bytes, wl.capacity_rows, plan=plan, order=order)
        c.fill()
        torch.cuda.synchronize()
        c.enable_timing(True)
        return c

    combos = [tuple(int(v) for v in c.split(":")) for c in args.combos.split(",") if c]
    cache = new_cache()
    batches = [torch.from_numpy(synth.make_batch(wl, 0, i)).cuda() for i in range(2)]
    n = batches[0].numel()
    out = torch.empty((n, wl.row_bytes), dtype=torch.uint8, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    cache.enable_timing(True)
    res = []
    for rows, warps in combos:
        os.environ["UGACHE_HOST_ROWS"] = str(rows)
        os.environ["UGACHE_HOST_WARPS"] = str(warps)
        c2 = new_cache()
        for hs in [int(x) for x in args.host_sms.split(",")]:
            c2.set_dedication(hs, 0)
            gms = []
            for r in range(args.reps + 1):
                flush.fill_(r)
                c2.extract(batches[r % 2], out)
                a, b = c2.last_batch_timing()
                if r:
                    gms.append(b)
            rec = {"rows": rows, "warps": warps, "host_sms": hs, "gather_ms": statistics.median(gms)}
            print(json.dumps(rec), flush=True)
        c2.close()
    for ordered in [int(x) for x in args.order.split(",")]:
        cache.set_host_ordering(bool(ordered))
        for hs in [int(x) for x in args.host_sms.split(",")]:
            cache.set_dedication(hs, 0)
            gms = []
            for r in range(args.reps + 1):
                flush.fill_(r)
                cache.extract(batches[r % 2], out)
                a, b = cache.last_batch_timing()
                if r:
                    gms.append(b)
            per, _ = cache.last_batch_stats()
            host_bytes = float(per[-1]) * wl.row_bytes
            g = statistics.median(gms)
            rec = {"ordered": ordered, "host_sms": hs, "gather_ms": g, "locate_ms": a,
                   "host_keys": int(per[-1]), "local_keys": int(per[0]),
                   "host_GBps_effective": host_bytes / (g * 1e-3) / 1e9}
            print(json.dumps(rec), flush=True)
            res.append(rec)
    if args.random:
        cache.set_mode("random")
        gms = []
        for r in range(args.reps + 1):
            flush.fill_(r)
            cache.extract(batches[r % 2], out)
            a, b = cache.last_batch_timing()
            if r:
                gms.append(b)
        print(json.dumps({"mode": "random", "gather_ms": statistics.median(gms)}), flush=True)
    if res:
        best = min(res, key=lambda x: x["gather_ms"])
        print(json.dumps({"best": best}), flush=True)


if __name__ == "__main__":
    main()
