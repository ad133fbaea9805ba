#!/usr/bin/env python3
"""Extraction paths with G fake peers on ONE B200 (G contexts on one device, each slab a
peer of the others): the two-phase factored kernel (K1 + grid barrier + K2), the single
pass (K3) with peer rows queued to dedicated SMs (default), K3 with peer rows copied inline
by the locating warps (no dedication), and unfactored random dispatch.

What it isolates: every "peer" row is local HBM here, so NVLink congestion -- what
dedication is for -- is absent; the numbers show each path's own overhead
(barrier, bucket traffic, queue claims) at the peer shares of a G-GPU placement.
Prints one JSON object (per G: ms per batch of GPU 0's batch, path, per-source keys).
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
    ap.add_argument("--workload", default="gnn_pa")
    ap.add_argument("--scale", type=float, default=0.1, help="row scale of the workload")
    ap.add_argument("--gpus", type=int, nargs="+", default=[2, 4, 8])
    ap.add_argument("--cache-ratio", type=float, default=0.2)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    import torch
    import synth
    from paper_conf_sosp_songz0c23_b200 import UGache, connect_in_process

    wl = synth.get_workload(args.workload)
    if args.scale != 1.0:
        wl = wl.scaled(args.scale)
    N, R = wl.num_rows, wl.row_bytes
    C = int(N * args.cache_ratio)
    table = synth.make_table(N, R)
    h = synth.hotness(wl)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    res = {"workload": wl.name, "num_rows": N, "row_bytes": R, "cache_ratio": args.cache_ratio,
           "keys_per_batch": wl.keys_per_batch, "runs": []}
    variants = {
        "two_phase": dict(mode="factored", stream="off", peers_inline=False),
        "single_pass_queued_peers": dict(mode="factored", stream="on", peers_inline=False),
        "single_pass_inline_peers": dict(mode="factored", stream="on", peers_inline=True),
        "random_dispatch": dict(mode="random", stream="off", peers_inline=False),
        "two_phase_4_peer_sms": dict(mode="factored", stream="off", peers_inline=False, peer_sms=4),
        "single_pass_queued_4_peer_sms": dict(mode="factored", stream="on", peers_inline=False, peer_sms=4),
    }
    for G in args.gpus:
        group = [UGache(table, N, R, C, hotness=h, num_gpus=G, rank=g, device=0) for g in range(G)]
        connect_in_process(group)
        for c in group:
            c.fill()
        torch.cuda.synchronize()
        c = group[0]
        keys_np = [synth.make_batch(wl, 0, b) for b in range(3)]
        keys = [torch.from_numpy(k).cuda() for k in keys_np]
        out = torch.empty((keys[0].numel(), R), dtype=torch.uint8, device="cuda")
        run = {"G": G, "variants": {}}
        for name, v in variants.items():
            c.set_mode(v["mode"])
            c.set_stream(v["stream"])
            c.set_inline(host=True, peers=v["peers_inline"])
            if G > 1:  # 0 = keep; the paper's default split is restored after the variant
                c.set_dedication(0, v.get("peer_sms", c.plan.peer_sms))
            ms = []
            for i in range(args.steps + 3):
                flush.fill_(i & 0xFF)
                torch.cuda._sleep(100_000)
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s.record()
                c.extract(keys[i % 3], out)
                e.record()
                torch.cuda.synchronize()
                if i >= 3:
                    ms.append(s.elapsed_time(e))
            ref = synth.rows_for_keys(keys_np[(args.steps + 2) % 3], N, R)   # the generator
            exact = bool(np.array_equal(out.cpu().numpy(), ref))
            per, _ = c.last_batch_stats()
            run["variants"][name] = {"ms": statistics.mean(ms), "path": c.last_extract_path(),
                                     "per_source": per.tolist(), "bit_exact": exact}
        res["runs"].append(run)
        print(json.dumps(run), file=sys.stderr, flush=True)
        for g in group:
            g.close()
    table.close()
    s = json.dumps(res, indent=1)
    print(s)
    if args.out:
        with open(args.out, "w") as f:
            f.write(s)


if __name__ == "__main__":
    main()
