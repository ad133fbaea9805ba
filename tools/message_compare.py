#!/usr/bin/env python3
"""Factored (peer loads) vs message-based (request/serve/reply) extraction on ONE B200 with
G fake peers (G contexts on one device, each slab a peer of the others).
row 1; P:617-733 (message-based), P:984-1103 (factored).

What it isolates: with fake peers every "peer" row is local HBM and every exchange is a
device copy, so the difference is the message design's own work -- a host sync for the
counts, packing the requests, a second pass over each peer row on the owner, a copy of
each reply, a scatter into key order -- not NVLink behaviour (one GPU only in this run).
Prints one JSON object.
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
    ap.add_argument("--scale", type=float, default=0.1, help="row scale of the workload")
    ap.add_argument("--gpus", type=int, nargs="+", default=[2, 4, 8])
    ap.add_argument("--cache-ratio", type=float, default=0.1)
    ap.add_argument("--policy", default="ugache")
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    import torch
    import synth
    from paper_conf_sosp_songz0c23_b200 import UGache, connect_in_process
    from paper_conf_sosp_songz0c23_b200.message import message_extract_group

    wl = synth.get_workload(args.workload)
    if args.scale != 1.0:
        wl = wl.scaled(args.scale)
    N, R = wl.num_rows, wl.row_bytes
    C = int(N * args.cache_ratio)
    table = synth.make_table(N, R)
    h = synth.hotness(wl)
    res = {"workload": wl.name, "num_rows": N, "row_bytes": R, "cache_ratio": args.cache_ratio,
           "policy": args.policy, "keys_per_batch": wl.keys_per_batch, "runs": []}
    for G in args.gpus:
        group = [UGache(table, N, R, C, hotness=h, num_gpus=G, rank=g, device=0, policy=args.policy)
                 for g in range(G)]
        connect_in_process(group)
        for c in group:
            c.fill()
        torch.cuda.synchronize()
        keys = [[torch.from_numpy(synth.make_batch(wl, g, b)).cuda() for g in range(G)] for b in range(2)]
        outs = [torch.empty((k.numel(), R), dtype=torch.uint8, device="cuda") for k in keys[0]]

        def factored(b):
            for g, c in enumerate(group):
                c.extract(keys[b][g], outs[g])

        def message(b):
            message_extract_group(group, keys[b], outs)

        row = {"G": G}
        for name, fn in (("factored", factored), ("message", message)):
            for w in range(3):
                fn(w % 2)
            torch.cuda.synchronize()
            ts = []
            for s in range(args.steps):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                t0 = time.perf_counter()
                e0.record()
                fn(s % 2)
                e1.record()
                torch.cuda.synchronize()
                ts.append(max(e0.elapsed_time(e1), (time.perf_counter() - t0) * 1e3))
            # parity of the last batch of every rank
            b = (args.steps - 1) % 2
            for g in range(G):
                ref = synth.rows_for_keys(keys[b][g].cpu().numpy(), N, R)   # the generator
                assert np.array_equal(outs[g].cpu().numpy(), ref), f"{name} G={G} rank {g} differs"
            row[f"{name}_ms_per_G_batches"] = statistics.mean(ts)
        per = [c.last_batch_stats()[0].tolist() for c in group]
        row["per_source_rank0"] = per[0]
        row["message_over_factored"] = row["message_ms_per_G_batches"] / row["factored_ms_per_G_batches"]
        res["runs"].append(row)
        print(json.dumps(row), file=sys.stderr, flush=True)
        for c in group:
            c.close()
        del outs, keys
        torch.cuda.empty_cache()
    s = json.dumps(res)
    print(s)
    if args.out:
        with open(args.out, "w") as f:
            f.write(s + "\n")


if __name__ == "__main__":
    main()
