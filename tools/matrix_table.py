#!/usr/bin/env python3
"""Markdown table of the bench lines in a directory (tools/config_matrix.sh)."""
import json
import os
import sys

d = sys.argv[1]
rows = []
for f in sorted(os.listdir(d)):
    if not f.endswith(".json"):
        continue
    try:
        j = json.loads(open(os.path.join(d, f)).read().strip().splitlines()[-1])
    except Exception as e:  # noqa: BLE001
        rows.append(f"| {f} | error: {e} |")
        continue
    c, r = j["config"], j["roofline"]
    ps = j["per_source_keys"]
    n = ps["local"] + ps["peer"] + ps["host"]
    ab = j.get("fem_ablation") or {}
    abc = ab.get("cold_l2") or {}
    ho = j.get("host_only") or {}
    cold = j.get("cold_l2") or {}
    rr = r.get("random_row_peak") or {}
    rows.append("| {} | {} | {:.0%} | {} | {:.4f} | {:.0f} | {} {:.2f} | {} | {:.4f} | {} | {} | {} | {} | {} |".format(
        c["workload"] + (f" (alpha {c['alpha']:g})" if c.get("alpha", 1.2) != 1.2 else ""),
        c["keys_per_batch_per_gpu"], c["cache_ratio"], r.get("path"), j["ms_per_step"], j["value"],
        r["term"], r["frac"], f"{rr['frac']:.2f}" if rr else "-",
        cold.get("ms_per_step", float("nan")), f"{cold['roofline_frac']:.2f}" if cold.get("roofline_frac") else "-",
        f"{ps['host'] / n:.1%}",
        f"{ab['random_dispatch_ms_per_step']:.4f}" if ab else "-",
        f"{abc['random_dispatch_ms_per_step']:.4f}" if abc else "-",
        f"{ho['ms']:.4f}" if ho else "-"))
print("| workload | keys/batch | c | path | ms/batch | GB/s | kernel roofline | vs random-row host peak "
      "| cold-L2 ms | cold-L2 frac | host share | random dispatch ms | random dispatch cold ms | host keys alone ms (cold) |")
print("|---|---|---|---|---|---|---|---|---|---|---|---|---|---|")
print("\n".join(rows))
