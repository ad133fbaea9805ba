#!/usr/bin/env python3
"""Back-to-back (steady-state) extraction diagnostics: per-step device time of K extracts
queued without host synchronisation, with and without CUDA events between steps, with a
short device spin between steps, with per-step host sync, and cycling 4 vs 8 distinct
batches.  Prints one JSON object per variant."""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="gnn_pa")
    ap.add_argument("--cache-ratio", type=float, default=None)
    ap.add_argument("--steps", type=int, default=20)
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
    cfg = make_config(wl.num_rows, wl.row_bytes, wl.capacity_rows, host_tier=True)
    plan, order = solve(cfg, h)
    del h
    cache = UGache(table, wl.num_rows, wl.row_bytes, wl.capacity_rows, plan=plan, order=order, host_tier=True)
    cache.fill()
    torch.cuda.synchronize()
    batches = [torch.from_numpy(synth.make_batch(wl, 0, i)).cuda() for i in range(16)]
    out = torch.empty((batches[0].numel(), wl.row_bytes), dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")

    def run(nb, events, gap_ns, sync, start, fl=False):
        for i in range(3):
            cache.extract(batches[(start + i) % nb], out, s)
        s.synchronize()
        evs = []
        t0 = torch.cuda.Event(enable_timing=True)
        t0.record(s)
        prev = t0
        for i in range(args.steps):
            if fl:
                with torch.cuda.stream(s):
                    flush.fill_(i & 0xFF)
            if gap_ns:
                with torch.cuda.stream(s):
                    torch.cuda._sleep(gap_ns)
            if events:
                b = torch.cuda.Event(enable_timing=True)
                b.record(s)
            cache.extract(batches[(start + 3 + i) % nb], out, s)
            e = torch.cuda.Event(enable_timing=True)
            e.record(s)
            if events:
                evs.append((b, e))
            prev = e
            if sync:
                s.synchronize()
        s.synchronize()
        tot = t0.elapsed_time(prev) / args.steps
        per = [a.elapsed_time(b) for a, b in evs]
        return {"nb": nb, "events": events, "gap": gap_ns, "sync": sync, "flush": fl,
                "ms_per_step_total": tot, "per_step": [round(x, 4) for x in per]}

    variants = [(8, True, 0, False, False), (8, False, 0, False, False), (4, False, 0, False, False),
                (8, True, 2000, False, False), (8, True, 20000, False, False), (8, True, 0, True, False),
                (16, True, 0, False, False), (8, True, 0, False, True)]
    for k, (nb, ev, gap, sync, fl) in enumerate(variants):
        print(json.dumps(run(nb, ev, gap, sync, k * 3, fl)), flush=True)
    cache.close()
    table.close()


if __name__ == "__main__":
    main()
