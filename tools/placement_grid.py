#!/usr/bin/env python3
"""BASELINE.json configs[4], the placement sweep: replication vs partition vs UGache through
the SAME kernels over cache ratio x Zipf alpha x G (Fig. 2 / Fig. 12 analog, P:385-413,
P:492-525), on ONE B200 with G fake peers.

Each (alpha, c, G, policy) point: G contexts on one device share one host table and a host
tier per placement; GPU 0 extracts distinct batches through the production path (auto
kernel choice), the first batch is compared with the table generator (tools never run the
oracle).  Same caveats as tools/policy_compare.py: host and local rows are read as on a real
node (except that GPU 0's host link serves only GPU 0), "peer" rows come from the other
contexts' slabs in the same HBM, so a peer-heavy placement's real time is at least
max(measured, NVLink ingress = peer bytes / 770 GB/s).

Replication's placement does not depend on G (every GPU holds the top C), so it is measured
once per (alpha, c) and reused for the other G; a UGache plan identical to partition (k = 0)
or to replication (k >= C) reuses that measurement (`same_as`).  One JSON line per point goes
to --out as it is measured, so a cut-off run keeps its points; --table writes the summary.
"""
from __future__ import annotations

import argparse
import dataclasses
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

NVL_GBS = 770.0


def table_md(rows, workload):
    """Markdown summary: one row per (alpha, c), one column group per G."""
    gs = sorted({r["G"] for r in rows})
    out = [f"# Placement sweep through the same kernels ({workload}, one B200, G fake peers)", "",
           "ms/batch of GPU 0 (cold L2, mean of the timed batches); peer-heavy placements are "
           "`max(measured, NVLink ingress)` = the lower bound a real node cannot beat; "
           "`k` = hot entries UGache replicates (0 = partition, C = replication).  All bit-exact "
           "unless marked.", ""]
    hdr = "| alpha | c |" + "".join(f" G={g} rep | G={g} part | G={g} ugache (k) | G={g} best |" for g in gs)
    out += [hdr, "|---|---|" + "---|---|---|---|" * len(gs)]
    keys = sorted({(r["alpha"], r["cache_ratio"]) for r in rows})
    for a, c in keys:
        line = f"| {a:g} | {c:g} |"
        for g in gs:
            pts = {r["policy"]: r for r in rows if r["alpha"] == a and r["cache_ratio"] == c and r["G"] == g}
            vals = {}
            for pol in ("replication", "partition", "ugache"):
                r = pts.get(pol)
                vals[pol] = r["lower_bound_ms"] if r else None
            cell = []
            for pol in ("replication", "partition", "ugache"):
                r = pts.get(pol)
                if not r:
                    cell.append("-")
                    continue
                s = f"{r['lower_bound_ms']:.3f}"
                if pol == "ugache":
                    s += f" ({r['k']})"
                if not r["bit_exact"]:
                    s += " MISMATCH"
                cell.append(s)
            have = {p: v for p, v in vals.items() if v is not None}
            best = min(have, key=have.get) if have else "-"
            line += "".join(f" {x} |" for x in cell) + f" {best} |"
        out.append(line)
    # ugache vs the better of the two baselines
    ratios = []
    for r in rows:
        if r["policy"] != "ugache":
            continue
        base = [q["lower_bound_ms"] for q in rows if q["G"] == r["G"] and q["alpha"] == r["alpha"]
                and q["cache_ratio"] == r["cache_ratio"] and q["policy"] != "ugache"]
        if len(base) == 2:
            ratios.append(min(base) / r["lower_bound_ms"])
    if ratios:
        out += ["", f"UGache speedup over the better of replication / partition (lower-bound times): "
                    f"min {min(ratios):.3f}x, median {statistics.median(ratios):.3f}x, max {max(ratios):.3f}x "
                    f"over {len(ratios)} points."]
    return "\n".join(out) + "\n"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="gnn_pa@0.25")
    ap.add_argument("--gpus", type=int, nargs="+", default=[2, 4, 8])
    ap.add_argument("--cache-ratios", type=float, nargs="+", default=[0.05, 0.1, 0.2, 0.5])
    ap.add_argument("--alphas", type=float, nargs="+", default=[0.8, 1.0, 1.2, 1.4])
    ap.add_argument("--policies", nargs="+", default=["replication", "partition", "ugache"])
    ap.add_argument("--steps", type=int, default=6)
    ap.add_argument("--out", default="")
    ap.add_argument("--table", default="")
    ap.add_argument("--summarize", default="", help="only rebuild --table from this JSONL file")
    ap.add_argument("--phases", action="store_true", help="record the fused kernel's phase stamps")
    ap.add_argument("--batch-n", type=int, default=0, help="override the workload's keys (or samples) per batch")
    ap.add_argument("--random", action="store_true",
                    help="also time random dispatch (unfactored) on the same contexts and batches")
    args = ap.parse_args()
    if args.summarize:
        rows = [json.loads(x) for x in open(args.summarize) if x.strip()]
        s = table_md(rows, args.workload)
        if args.table:
            open(args.table, "w").write(s)
        print(s)
        return
    import torch
    import synth
    from paper_conf_sosp_songz0c23_b200 import (UGache, connect_in_process, fill_host_tier,
                                                host_tier_rows, make_config, solve)
    wl0 = synth.get_workload(args.workload)
    N, R = wl0.num_rows, wl0.row_bytes
    torch.cuda.set_device(0)
    table = synth.HostTable(N, R)
    table.fill()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    fout = open(args.out, "a") if args.out else None
    rows = []
    nb = args.steps + 2
    for alpha in args.alphas:
        wl = dataclasses.replace(wl0, alpha=alpha)
        if args.batch_n:
            wl = dataclasses.replace(wl, batch_n=args.batch_n)
        t0 = time.time()
        h = synth.hotness(wl)
        keys_np = [synth.make_batch(wl, 0, b) for b in range(nb)]
        keys = [torch.from_numpy(k).cuda() for k in keys_np]
        ref0 = synth.rows_for_keys(keys_np[0], N, R)
        out = torch.empty((keys[0].numel(), R), dtype=torch.uint8, device="cuda")
        print(f"[grid] alpha {alpha}: hotness + {nb} batches in {time.time() - t0:.1f}s", file=sys.stderr)
        for c_ratio in args.cache_ratios:
            C = int(round(N * c_ratio))
            done = {}   # placement signature -> measured row
            for G in args.gpus:
                for pol in args.policies:
                    cfg = make_config(N, R, C, num_gpus=G, policy=pol, host_tier=True)
                    plan, order = solve(cfg, h)
                    sig = ("replication",) if (pol == "replication" or (pol == "ugache" and plan.k >= C)) \
                        else (G, int(plan.k), int(plan.band_end))
                    base = {"alpha": alpha, "cache_ratio": c_ratio, "G": G, "policy": pol, "k": int(plan.k),
                            "band_end": int(plan.band_end), "model_z_ms": plan.z * 1e3}
                    if sig in done:
                        r = dict(done[sig], **base)
                        r["same_as"] = f"{done[sig]['policy']} G={done[sig]['G']}"
                        r["model_z_ms"] = plan.z * 1e3
                    else:
                        t1 = time.time()
                        tier = synth.HostTable(host_tier_rows(plan, N), R)
                        fill_host_tier(cfg, order, plan, table, tier)
                        group = [UGache(table, N, R, C, num_gpus=G, rank=g, device=0, policy=pol, plan=plan,
                                        order=order, host_tier=tier) for g in range(G)]
                        connect_in_process(group)
                        for cc in group:
                            cc.fill()
                        torch.cuda.synchronize()
                        cc = group[0]
                        cc.enable_timing(args.phases)
                        ms, phases = [], []
                        for i in range(nb):
                            flush.fill_(i & 0xFF)
                            torch.cuda._sleep(100_000)
                            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                            s.record()
                            cc.extract(keys[i], out)
                            e.record()
                            torch.cuda.synchronize()
                            if i >= 2:
                                ms.append(s.elapsed_time(e))
                                if args.phases:
                                    try:
                                        phases.append([round(x, 4) for x in cc.last_batch_phases()])
                                    except Exception:  # noqa: BLE001 - single pass has no stamps
                                        phases.append(None)
                        path = cc.last_extract_path()
                        rnd = []
                        if args.random:
                            cc.set_mode("random")
                            for i in range(nb):
                                flush.fill_(i & 0xFF)
                                torch.cuda._sleep(100_000)
                                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                                s.record()
                                cc.extract(keys[i], out)
                                e.record()
                                torch.cuda.synchronize()
                                if i >= 2:
                                    rnd.append(s.elapsed_time(e))
                            cc.set_mode("factored")
                        cc.extract(keys[0], out)
                        torch.cuda.synchronize()
                        exact = bool(np.array_equal(out.cpu().numpy(), ref0))
                        per, _ = cc.last_batch_stats()
                        n = int(per.sum())
                        n_peer = int(per.sum() - per[0] - per[G])
                        nvl_ms = n_peer * R / (NVL_GBS * 1e9) * 1e3
                        meas = statistics.mean(ms)
                        r = dict(base, share={"local": per[0] / n, "peer": n_peer / n, "host": per[G] / n},
                                 measured_ms=meas, ms=ms, path=path, bit_exact=exact,
                                 nvlink_ingress_ms=nvl_ms, lower_bound_ms=max(meas, nvl_ms),
                                 setup_s=time.time() - t1)
                        if args.phases:
                            r["phases_ms"] = phases
                        if rnd:
                            r["random_dispatch_ms"] = statistics.mean(rnd)
                        done[sig] = r
                        for g in group:
                            g.close()
                        tier.close()
                        del group
                        torch.cuda.empty_cache()
                    rows.append(r)
                    line = json.dumps(r)
                    print(line, file=sys.stderr, flush=True)
                    if fout:
                        fout.write(line + "\n")
                        fout.flush()
    table.close()
    s = table_md(rows, wl0.name)
    if args.table:
        open(args.table, "w").write(s)
    print(s)


if __name__ == "__main__":
    main()
