#!/usr/bin/env python3
"""Per-role timeline of the fused kernel (ugache_last_batch_timeline): for each role (host,
each peer, local) the number of CTAs and the median / max of gather start, role done and
CTA done, in us from the kernel's start -- the paper's Fig. 8 picture of one batch
(P:1086-1103).  gnn_pa@0.25 table, UGache placement, G fake peers, batches back to back
(steady state), the last one reported.  Also writes the raw per-CTA rows (--out)."""
from __future__ import annotations

import argparse
import dataclasses
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402


def summarize(tl, G, rank=0):
    roles = {}
    for row in tl:
        src = int(row[0])
        name = "host" if src == G else "mixed" if src == G + 1 else ("local" if src == rank else f"peer{src}")
        roles.setdefault(name, []).append(row)
    out = {}
    for name, rows in sorted(roles.items()):
        a = np.array(rows)
        out[name] = {"ctas": len(rows),
                     "cta_start_us": [round(float(np.median(a[:, 1])) * 1e3, 2), round(float(a[:, 1].max()) * 1e3, 2)],
                     "gather_start_us": [round(float(np.median(a[:, 2])) * 1e3, 2), round(float(a[:, 2].max()) * 1e3, 2)],
                     "role_done_us": [round(float(np.median(a[:, 3])) * 1e3, 2), round(float(a[:, 3].max()) * 1e3, 2)],
                     "cta_done_us": [round(float(np.median(a[:, 4])) * 1e3, 2), round(float(a[:, 4].max()) * 1e3, 2)]}
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="gnn_pa@0.25")
    ap.add_argument("--gpus", type=int, nargs="+", default=[4])
    ap.add_argument("--batch-n", type=int, nargs="+", default=[2000, 100000, 500000])
    ap.add_argument("--cache-ratio", type=float, default=0.2)
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    import torch
    import synth
    from paper_conf_sosp_songz0c23_b200 import (UGache, connect_in_process, fill_host_tier,
                                                host_tier_rows, make_config, solve)
    wl0 = synth.get_workload(args.workload)
    N, R = wl0.num_rows, wl0.row_bytes
    C = int(round(N * args.cache_ratio))
    torch.cuda.set_device(0)
    table = synth.HostTable(N, R)
    table.fill()
    h = synth.hotness(wl0)
    raw = []
    for G in args.gpus:
        cfg = make_config(N, R, C, num_gpus=G, policy="ugache", host_tier=True)
        plan, order = solve(cfg, h)
        tier = synth.HostTable(host_tier_rows(plan, N), R)
        fill_host_tier(cfg, order, plan, table, tier)
        group = [UGache(table, N, R, C, num_gpus=G, rank=g, device=0, policy="ugache", plan=plan,
                        order=order, host_tier=tier) for g in range(G)]
        connect_in_process(group)
        for cc in group:
            cc.fill()
        torch.cuda.synchronize()
        c = group[0]
        c.set_stream("off")
        c.enable_timing(True)
        for n in args.batch_n:
            wl = dataclasses.replace(wl0, batch_n=n)
            keys = [torch.from_numpy(synth.make_batch(wl, 0, b)).cuda() for b in range(4)]
            out = torch.empty((n, R), dtype=torch.uint8, device="cuda")
            for i in range(12):
                c.extract(keys[i % 4], out)
            tl = c.last_batch_timeline()
            per, _ = c.last_batch_stats()
            r = {"G": G, "n": n, "per_source": per.tolist(), "phases_ms": c.last_batch_phases(),
                 "roles": summarize(tl, G)}
            print(json.dumps(r), flush=True)
            raw.append({"G": G, "n": n, "timeline_ms": tl.tolist()})
        for cc in group:
            cc.close()
        tier.close()
        del group
        torch.cuda.empty_cache()
    if args.out:
        json.dump(raw, open(args.out, "w"))
    table.close()


if __name__ == "__main__":
    main()
