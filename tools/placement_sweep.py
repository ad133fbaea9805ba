#!/usr/bin/env python3
"""Placement sweep (BASELINE.json configs[4]): replication vs partition vs the UGache policy
on the same model and location tables, for cache ratio c, Zipf alpha and G GPUs.

For each setting it solves all three policies with ugache_solve (host only), builds GPU 0's
location table with ugache_build_placement, and reports the expected share of GPU 0's
accesses served locally / by peers / by the host (hotness-mass fractions, exact), the
replicated prefix k/C and the section 6.2 modeled batch time z.  PA-shaped
rows scaled to --rows (default 2M) with a 500K-unique-per-111M-equivalent batch.
Writes a markdown table (and JSON) to --out.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rows", type=int, default=2_000_000)
    ap.add_argument("--gpus", default="2,4,8")
    ap.add_argument("--cache", default="0.02,0.05,0.1,0.2,0.3,0.5")
    ap.add_argument("--alpha", default="0.8,1.0,1.2,1.4")
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r1", "placement_sweep"))
    args = ap.parse_args()
    import synth
    from paper_conf_sosp_songz0c23_b200 import build_placement, make_config, solve

    N = args.rows
    rows = []
    for alpha in [float(a) for a in args.alpha.split(",")]:
        wl = synth.Workload("sweep", (N,), 512, alpha, "unique", max(1, N * 500_000 // 111_000_000))
        h = synth.hotness(wl)
        hh = h.astype(np.float64)
        tot = hh.sum()
        for G in [int(g) for g in args.gpus.split(",")]:
            for c in [float(x) for x in args.cache.split(",")]:
                C = int(round(c * N))
                rec = {"alpha": alpha, "G": G, "c": c}
                for pol in ("replication", "partition", "ugache"):
                    cfg = make_config(N, 512, C, num_gpus=G, policy=pol)
                    plan, order = solve(cfg, h)
                    loc, _ = build_placement(cfg, order, plan, 0)
                    src = (loc >> np.uint64(56)).astype(np.int64)
                    mass = np.bincount(src, weights=hh, minlength=G + 1) / tot
                    rec[pol] = {"local": float(mass[0]), "peer": float(mass[1:G].sum()),
                                "host": float(mass[G]), "k_over_C": plan.k / max(C, 1),
                                "z_us": plan.z * 1e6}
                rows.append(rec)
                u, r_, p_ = rec["ugache"], rec["replication"], rec["partition"]
                print(f"a={alpha} G={G} c={c:.2f}: z rep {r_['z_us']:.1f} part {p_['z_us']:.1f} "
                      f"ugache {u['z_us']:.1f} us (k/C {u['k_over_C']:.3f}, local {u['local']:.3f} "
                      f"peer {u['peer']:.3f} host {u['host']:.3f})", flush=True)
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out + ".json", "w") as f:
        json.dump({"rows": N, "results": rows}, f, indent=1)
    with open(args.out + ".md", "w") as f:
        f.write(f"# Placement sweep (model, GPU 0 of G; PA-shaped {N:,} rows x 512 B, "
                f"unique batches)\n\nShares are expected fractions of GPU 0's accesses; z is the "
                f"section 6.2 modeled batch time with the library's default B200 parameters.\n\n")
        f.write("| alpha | G | c | z rep (us) | z part (us) | z ugache (us) | ugache/min(rep,part) | "
                "ugache k/C | ugache local / peer / host | part local / peer / host |\n")
        f.write("|---|---|---|---|---|---|---|---|---|---|\n")
        for r in rows:
            u, rp, pp = r["ugache"], r["replication"], r["partition"]
            best = min(rp["z_us"], pp["z_us"])
            f.write(f"| {r['alpha']} | {r['G']} | {r['c']:.2f} | {rp['z_us']:.1f} | {pp['z_us']:.1f} | "
                    f"{u['z_us']:.1f} | {u['z_us'] / best:.3f} | {u['k_over_C']:.3f} | "
                    f"{u['local']:.3f} / {u['peer']:.3f} / {u['host']:.3f} | "
                    f"{pp['local']:.3f} / {pp['peer']:.3f} / {pp['host']:.3f} |\n")
    print("wrote", args.out + ".md")


if __name__ == "__main__":
    main()
