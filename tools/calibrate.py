#!/usr/bin/env python3
"""A0 calibration on one B200 (Fig. 6 analog): factored-gather time vs the
number of SMs dedicated to the host source, on a real workload placement, for a list of
environment settings (UGACHE_HOST_WARPS, UGACHE_HOST_SORT_MIN, UGACHE_HOST_DYNAMIC, ...),
each in a fresh context.  Prints one JSON object per measurement and the best setting.

  python tools/calibrate.py --workload gnn_pa --host-sms 4,8,12,16 \
      --env "UGACHE_HOST_DYNAMIC=0;UGACHE_HOST_DYNAMIC=0 UGACHE_HOST_SORT_MIN=0" --random
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="gnn_pa")
    ap.add_argument("--cache-ratio", type=float, default=None)
    ap.add_argument("--host-sms", default="2,4,8,12,16,24,32,48")
    ap.add_argument("--reps", type=int, default=6)
    ap.add_argument("--env", default="", help="';'-separated settings, each 'K=V K=V'")
    ap.add_argument("--order", default="1", help="host ordering values to sweep, e.g. 1,0")
    ap.add_argument("--host-tier", action="store_true")
    ap.add_argument("--random", action="store_true", help="also time random dispatch")
    ap.add_argument("--batches", type=int, default=4, help="distinct batches cycled (>= 4: no warm host translations)")
    ap.add_argument("--warp-host", default="", help="also sweep warp-granular dedication: host warps per SM, e.g. 1,2,4")
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
    batches = [torch.from_numpy(synth.make_batch(wl, 0, i)).cuda() for i in range(args.batches)]
    n = batches[0].numel()
    out = torch.empty((n, wl.row_bytes), dtype=torch.uint8, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")

    def new_cache():
        c = UGache(table, wl.num_rows, wl.row_bytes, wl.capacity_rows, plan=plan, order=order,
                   host_tier=args.host_tier)
        c.fill()
        torch.cuda.synchronize()
        c.enable_timing(True)
        return c

    def timed(c):
        gms = []
        for r in range(args.reps + 1):
            flush.fill_(r)
            c.extract(batches[r % len(batches)], out)
            _, b = c.last_batch_timing()
            if r:
                gms.append(b)
        return statistics.median(gms)

    settings = [s for s in args.env.split(";")] if args.env else [""]
    res = []
    for setting in settings:
        saved = dict(os.environ)
        for kv in setting.split():
            k, v = kv.split("=", 1)
            os.environ[k] = v
        c = new_cache()
        for ordered in [int(x) for x in args.order.split(",")]:
            c.set_host_ordering(bool(ordered))
            for hs in [int(x) for x in args.host_sms.split(",")]:
                c.set_dedication(hs, 0)
                g = timed(c)
                per, _ = c.last_batch_stats()
                rec = {"env": setting, "ordered": ordered, "host_sms": hs, "gather_ms": g,
                       "host_keys": int(per[-1]), "local_keys": int(per[0]),
                       "host_GBps_effective": float(per[-1]) * wl.row_bytes / (g * 1e-3) / 1e9}
                print(json.dumps(rec), flush=True)
                res.append(rec)
        for hw in [int(x) for x in args.warp_host.split(",") if x]:
            c.set_dedication_mode("warps", host_warps=hw)
            for ordered in [int(x) for x in args.order.split(",")]:
                c.set_host_ordering(bool(ordered))
                g = timed(c)
                per, _ = c.last_batch_stats()
                rec = {"env": setting, "dedication": "warps", "host_warps_per_sm": hw,
                       "ordered": ordered, "gather_ms": g, "host_keys": int(per[-1]),
                       "host_GBps_effective": float(per[-1]) * wl.row_bytes / (g * 1e-3) / 1e9}
                print(json.dumps(rec), flush=True)
                res.append(rec)
            c.set_dedication_mode("sms")
        if args.random and setting == settings[0]:
            c.set_mode("random")
            print(json.dumps({"mode": "random", "gather_ms": timed(c)}), flush=True)
        c.close()
        os.environ.clear()
        os.environ.update(saved)
    best = min(res, key=lambda x: x["gather_ms"])
    print(json.dumps({"best": best}), flush=True)


if __name__ == "__main__":
    main()
