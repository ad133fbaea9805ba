#!/usr/bin/env python3
"""Cache-refresh timeline on one B200 (Fig. 17 analog; section 7.2).

The hotness drifts (a fraction of the cached hot set is replaced), foreground extraction
keeps running, and the Refresher applies the new placement.  --protocol chunked (default):
stage, then per slot range of --chunk slots: evict (that range's changing keys -> host),
one foreground batch, fill (throttled to --max-sms SMs, in --fill-rows sub-steps with a
foreground batch after each), install; then commit -- only one range's keys are ever
redirected to the host.  --protocol whole: begin (every changing key -> host), chunked
content rewrite with a foreground batch after every chunk, commit.  The ctx runs the
shipped configuration (host tier on, ugache_init from the old hotness).  Prints one JSON
object with the per-batch foreground times labelled by phase and the refresh duration.
"""
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
    ap.add_argument("--shift", type=float, default=0.5, help="fraction of the cached set replaced")
    ap.add_argument("--chunk", type=int, default=262144)
    ap.add_argument("--fill-rows", type=int, default=65536)
    ap.add_argument("--protocol", default="chunked", choices=["chunked", "whole"])
    ap.add_argument("--no-host-tier", dest="host_tier", action="store_false", default=True)
    ap.add_argument("--max-sms", type=int, default=16)
    ap.add_argument("--batches", type=int, default=20)
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    import torch
    import synth
    from paper_conf_sosp_songz0c23_b200 import UGache
    from paper_conf_sosp_songz0c23_b200.refresh import modeled_time, plan_placements

    wl = synth.get_workload(args.workload)
    N, R, C = wl.num_rows, wl.row_bytes, wl.capacity_rows
    torch.cuda.set_device(0)
    table = synth.HostTable(N, R)
    table.fill()
    h1 = synth.hotness(wl)
    order1 = np.argsort(-h1.astype(np.float64), kind="stable")
    # drift: the ranks [C*(1-shift), C) swap places with the ranks just beyond C
    s = int(C * args.shift)
    order2 = order1.copy()
    order2[C - s:C], order2[C:C + s] = order1[C:C + s].copy(), order1[C - s:C].copy()
    h2 = np.empty_like(h1)
    h2[order2] = np.sort(h1)[::-1]
    kw = dict(num_rows=N, row_bytes=R, capacity_rows=C)
    plan1, (pl1,) = plan_placements(kw, h1, 1)
    plan2, (pl2,) = plan_placements(kw, h2, 1)
    if args.host_tier:
        cache = UGache(table, N, R, C, hotness=h1, host_tier=True)
    else:
        cache = UGache(table, N, R, C, placement=pl1)
    cache.fill()
    torch.cuda.synchronize()
    cache.enable_timing(True)
    # foreground batches drawn from the drifted distribution (ranks mapped through order2)
    batches = []
    for b in range(4):
        k = synth.make_batch(wl, 0, b)
        ranks = synth.key_to_rank(k, N)
        batches.append(torch.from_numpy(order2[ranks].astype(np.int64)).cuda())
    n = batches[0].numel()
    out = torch.empty((n, R), dtype=torch.uint8, device="cuda")
    timeline = []
    i = [0]

    def fg(phase):
        cache.extract(batches[i[0] % len(batches)], out)
        a, g = cache.last_batch_timing()
        per, _ = cache.last_batch_stats()
        timeline.append({"phase": phase, "t_ms": (time.perf_counter() - t0) * 1e3, "gather_ms": a + g,
                         "host_keys": int(per[1])})
        i[0] += 1

    t0 = time.perf_counter()
    for _ in range(args.batches):
        fg("before")
    tr0 = time.perf_counter()
    chunks = []
    if args.protocol == "whole":
        cache.refresh_begin(*pl2)
        fg("evicted")
        while True:
            tc = time.perf_counter()
            rem = cache.refresh_content(args.max_sms, args.chunk)
            torch.cuda.synchronize()
            chunks.append((time.perf_counter() - tc) * 1e3)
            fg("content")
            if rem == 0:
                break
    else:
        cache.refresh_stage(*pl2)
        for lo in range(0, C, args.chunk):
            hi = min(C, lo + args.chunk)
            cache.refresh_chunk("evict", lo, hi)
            fg("evicted")                      # the batch between hashtable and content update
            for a in range(lo, hi, args.fill_rows):
                tc = time.perf_counter()
                cache.refresh_chunk("fill", a, min(hi, a + args.fill_rows), args.max_sms)
                torch.cuda.synchronize()
                chunks.append((time.perf_counter() - tc) * 1e3)
                fg("content")
            cache.refresh_chunk("install", lo, hi)
    cache.refresh_commit()
    tr1 = time.perf_counter()
    for _ in range(args.batches):
        fg("after")
    by = {}
    for r in timeline:
        by.setdefault(r["phase"], []).append(r["gather_ms"])
    res = {"workload": wl.name, "shift": args.shift, "chunk_rows": args.chunk, "max_sms": args.max_sms,
           "protocol": args.protocol, "host_tier": args.host_tier, "fill_rows": args.fill_rows,
           "changed_slots": int(np.sum(pl1[1] != pl2[1])), "refresh_ms": (tr1 - tr0) * 1e3,
           "content_chunks": len(chunks), "content_chunk_ms_mean": statistics.mean(chunks),
           "gather_ms_mean": {k: statistics.mean(v) for k, v in by.items()},
           "during_over_before": statistics.mean(by.get("evicted", []) + by.get("content", [])) /
                                 statistics.mean(by["before"]),
           "worst_over_before": max(by.get("evicted", []) + by.get("content", [])) / statistics.mean(by["before"]),
           "model_z_us": {"old_placement_new_hotness": modeled_time([pl1[0]], h2, plan2) * 1e6,
                          "new_placement_new_hotness": plan2.z * 1e6},
           "timeline": timeline}
    print(json.dumps({k: v for k, v in res.items() if k != "timeline"}))
    if args.out:
        with open(args.out, "w") as f:
            json.dump(res, f, indent=1)
    cache.close()
    table.close()


if __name__ == "__main__":
    main()
