#!/usr/bin/env python3
"""Replication vs partition vs UGache through the same kernels (Fig. 2 / Fig. 12 analog,
P:385-413) on ONE B200 with G fake peers.

For each G and policy: G contexts on one device share the full-size host table (and one
host tier per policy, built once), GPU 0 extracts its own batches through the production
path (auto: fused two-phase kernel with dedicated host / peer SMs), bit-exact against the
table generator.  What one GPU can and cannot show:
  * host rows and local rows are read exactly as on a real node (the host link of GPU 0
    serves only GPU 0 here; on a node all G GPUs read host memory at once);
  * "peer" rows come from the other contexts' slabs in the SAME HBM, i.e. faster than NVLink:
    the measured time is a lower bound for peer-heavy placements, and the NVLink ingress
    term (peer bytes / 770 GB/s, B200_PROFILING.md) is the other lower bound.
So: for replication (no peer rows) the measurement is the real single-GPU-link time; for
partition / UGache the real time is at least max(measured, NVLink ingress).  Prints one
JSON object per (G, policy) and a summary table.
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

NVL_GBS = 770.0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="gnn_pa")
    ap.add_argument("--gpus", type=int, nargs="+", default=[2, 4, 8])
    ap.add_argument("--cache-ratio", type=float, default=0.1)
    ap.add_argument("--policies", nargs="+", default=["replication", "partition", "ugache"])
    ap.add_argument("--steps", type=int, default=8)
    ap.add_argument("--no-host-tier", dest="host_tier", action="store_false", default=True)
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    import torch
    import synth
    from paper_conf_sosp_songz0c23_b200 import (UGache, connect_in_process, fill_host_tier,
                                                host_tier_rows, make_config, solve)
    wl = synth.get_workload(args.workload)
    N, R = wl.num_rows, wl.row_bytes
    C = int(round(N * args.cache_ratio))
    torch.cuda.set_device(0)
    table = synth.HostTable(N, R)
    table.fill()
    h = synth.hotness(wl)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    keys_np = [synth.make_batch(wl, 0, b) for b in range(3)]
    keys = [torch.from_numpy(k).cuda() for k in keys_np]
    out = torch.empty((keys[0].numel(), R), dtype=torch.uint8, device="cuda")
    ref0 = synth.rows_for_keys(keys_np[0], N, R)   # the table generator (tools never run the oracle)
    rows = []
    for G in args.gpus:
        for pol in args.policies:
            cfg = make_config(N, R, C, num_gpus=G, policy=pol, host_tier=args.host_tier)
            plan, order = solve(cfg, h)
            tier = False
            if args.host_tier:
                tier = synth.HostTable(host_tier_rows(plan, N), R)
                fill_host_tier(cfg, order, plan, table, tier)
            group = [UGache(table, N, R, C, num_gpus=G, rank=g, device=0, policy=pol, plan=plan,
                            order=order, host_tier=tier) for g in range(G)]
            connect_in_process(group)
            for c in group:
                c.fill()
            torch.cuda.synchronize()
            c = group[0]
            ms = []
            for i in range(args.steps + 2):
                flush.fill_(i & 0xFF)
                torch.cuda._sleep(100_000)
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s.record()
                c.extract(keys[i % 3], out)
                e.record()
                torch.cuda.synchronize()
                if i >= 2:
                    ms.append(s.elapsed_time(e))
            c.extract(keys[0], out)
            torch.cuda.synchronize()
            exact = bool(np.array_equal(out.cpu().numpy(), ref0))
            per, _ = c.last_batch_stats()
            n = int(per.sum())
            n_peer = int(per.sum() - per[0] - per[G])
            nvl_ms = n_peer * R / (NVL_GBS * 1e9) * 1e3
            meas = statistics.mean(ms)
            r = {"G": G, "policy": pol, "k": int(plan.k), "band_end": int(plan.band_end),
                 "share": {"local": per[0] / n, "peer": n_peer / n, "host": per[G] / n},
                 "measured_ms": meas, "path": c.last_extract_path(), "bit_exact": exact,
                 "nvlink_ingress_ms": nvl_ms, "lower_bound_ms": max(meas, nvl_ms),
                 "model_z_ms": plan.z * 1e3}
            rows.append(r)
            print(json.dumps(r), file=sys.stderr, flush=True)
            for g in group:
                g.close()
            if isinstance(tier, synth.HostTable):
                tier.close()
            del group
            torch.cuda.empty_cache()
    res = {"workload": wl.name, "cache_ratio": args.cache_ratio, "host_tier": args.host_tier,
           "keys_per_batch": wl.keys_per_batch, "nvlink_gbs": NVL_GBS, "rows": rows}
    s = json.dumps(res, indent=1)
    print(s)
    if args.out:
        with open(args.out, "w") as f:
            f.write(s)
    table.close()


if __name__ == "__main__":
    main()
