#!/usr/bin/env python3
"""Fig. 16 analog: the library's cache policies against the
optimal cache of the section 6.2 MILP solved at entry granularity, on reduced instances.

Not a test (not collected): a report script kept with the tests because it runs the oracle
(oracle/milp.py, the entry-level MILP with HiGHS, time-limited) next to the two product
solvers -- the hot-replicate / warm-partition sweep of ugache_solve (the default) and the
block-level MILP of milp_solver.py (section 6.3) -- under the same platform model (B200
parameters of DESIGN.md R11, 12 host SMs).  Writes profiles/r2/solver_gap.{md,json}.
The paper reports a 1.9 % average gap between UGache's policy and the optimum.
"""
from __future__ import annotations

import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import synth  # noqa: E402
from oracle import milp  # noqa: E402
from oracle.placement import Platform, rank_order  # noqa: E402
from paper_conf_sosp_songz0c23_b200 import make_config, solve  # noqa: E402
from paper_conf_sosp_songz0c23_b200.milp_solver import make_blocks, solve_blocks  # noqa: E402

BW = dict(bw_local=6457.7e9, bw_peer=770e9, bw_host=34.4e9)
HOST_SMS = 12


def instance(E, G, c, alpha, seed, time_limit):
    h = (synth.zipf_pmf(E, alpha) * 8192).astype(np.float32)[np.random.default_rng(seed).permutation(E)]
    C = max(1, int(round(c * E)))
    cfg = make_config(E, 512, C, num_gpus=G, host_sms=HOST_SMS, **BW)
    plan, order = solve(cfg, h)
    plat = Platform(G=G, row_bytes=512, host_sms=HOST_SMS, peer_sms=int(plan.peer_sms),
                    num_sms=int(plan.num_sms), **BW)
    t0 = time.time()
    opt = milp.solve(h, C, plat, time_limit=time_limit)
    t_opt = time.time() - t0
    hs = h[rank_order(h, E)]
    blocks = make_blocks(hs, G)
    T = (plan.T_local, plan.T_peer, plan.T_host)
    Rr = (plan.R_local, plan.R_peer, plan.R_host)
    _, _, z_block, _ = solve_blocks(hs, blocks, C, G, T, Rr, time_limit=time_limit)
    return {"E": E, "G": G, "cache_ratio": c, "C": C, "alpha": alpha,
            "z_opt_us": opt["z"] * 1e6, "opt_mip_gap": opt["mip_gap"], "opt_seconds": t_opt,
            "opt_status": int(opt["status"]),
            "z_sweep_us": plan.z * 1e6, "k": int(plan.k),
            "z_block_us": z_block * 1e6, "blocks": len(blocks),
            "z_replication_us": plan.z_replication * 1e6, "z_partition_us": plan.z_partition * 1e6,
            "gap_sweep": plan.z / opt["z"] - 1, "gap_block": z_block / opt["z"] - 1}


def main():
    time_limit = float(os.environ.get("GAP_TIME_LIMIT", "60"))
    cases = []
    for G in (2, 4, 8):
        for E in {2: (60, 120, 240), 4: (40, 60, 120, 240), 8: (24, 40)}[G]:
            for c in (0.05, 0.1, 0.2):
                for alpha in (1.2, 1.4):
                    cases.append((E, G, c, alpha))
    rows = []
    for i, (E, G, c, alpha) in enumerate(cases):
        r = instance(E, G, c, alpha, seed=i, time_limit=time_limit)
        rows.append(r)
        print(json.dumps(r), flush=True)
    out = os.path.join(ROOT, "profiles", "r2", "solver_gap")
    os.makedirs(os.path.dirname(out), exist_ok=True)
    with open(out + ".json", "w") as f:
        json.dump({"time_limit_s": time_limit, "host_sms": HOST_SMS, "bw": BW, "rows": rows}, f, indent=1)
    lines = ["# Fig. 16 analog: library policies vs the entry-level MILP optimum (section 6.2 model)",
             "",
             f"Reduced instances, Zipf hotness, B200 model parameters (DESIGN.md R11), {HOST_SMS} host SMs; "
             f"HiGHS time limit {time_limit:g} s per MILP (mip gap column: the optimum's own certified "
             "gap when the limit was hit).  gap = z / z_opt - 1.  Written by tests/report_solver_gap.py.",
             "",
             "| E | G | c | alpha | z_opt (us) | opt mip gap | sweep z (us) | sweep gap | block MILP z (us) | block gap | replication | partition |",
             "|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for r in rows:
        lines.append(f"| {r['E']} | {r['G']} | {r['cache_ratio']:g} | {r['alpha']:g} | {r['z_opt_us']:.4f} | "
                     f"{(r['opt_mip_gap'] or 0):.2%} | {r['z_sweep_us']:.4f} | {r['gap_sweep']:+.2%} | "
                     f"{r['z_block_us']:.4f} | {r['gap_block']:+.2%} | {r['z_replication_us']:.4f} | "
                     f"{r['z_partition_us']:.4f} |")
    gs = [r["gap_sweep"] for r in rows]
    gb = [r["gap_block"] for r in rows]
    lines += ["", f"Mean gap: sweep {np.mean(gs):+.2%} (max {np.max(gs):+.2%}); block MILP {np.mean(gb):+.2%} "
              f"(max {np.max(gb):+.2%}).  Paper (its block method vs optimal, measured): 1.9 % on average."]
    with open(out + ".md", "w") as f:
        f.write("\n".join(lines) + "\n")
    print("\n".join(lines[-1:]))


if __name__ == "__main__":
    main()
