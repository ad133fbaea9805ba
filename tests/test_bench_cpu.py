"""bench.py's reference arm (the CPU oracle, no GPU): the JSON-line contract on the tiny
config, and that non-zero ranks of a multi-rank launch exit 0 without output."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(extra_env):
    env = dict(os.environ, **extra_env)
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                           "--workload", "tiny", "--steps", "2", "--warmup", "3"],
                          cwd=ROOT, env=env, capture_output=True, text=True, timeout=300)


def test_reference_arm_json_line():
    r = _run({"RANK": "0", "WORLD_SIZE": "1", "LOCAL_RANK": "0"})
    assert r.returncode == 0, r.stderr
    lines = [l for l in r.stdout.splitlines() if l.strip()]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference"
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
              "higher_is_better", "scaling", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["steps"] == 2 and d["warmup"] == 3 and d["value"] > 0 and d["unit"] == "GB/s"
    assert d["config"]["workload"] == "tiny"
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["cpu_baseline"]["value"] == d["value"]
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0


def test_reference_arm_nonzero_rank_is_silent():
    r = _run({"RANK": "1", "WORLD_SIZE": "2", "LOCAL_RANK": "1"})
    assert r.returncode == 0, r.stderr
    assert r.stdout.strip() == ""


def test_batch_roofline_hand_computed():
    """bench.batch_roofline on a 2-GPU batch worked by hand (SURVEY.md 8(d) terms): HBM bytes
    include the rows served to the peer, NVLink egress = those rows, T_roof = max over GPUs."""
    sys.path.insert(0, ROOT)
    import bench
    R, kb = 512, 8
    # GPU0 reads 600 local, 300 from GPU1, 100 host; GPU1 reads 500 local, 200 from GPU0, 300 host
    P = [[600, 300, 100], [200, 500, 300]]
    n = [1000, 1000]
    rl = bench.batch_roofline(P, n, R, kb, "fused", hbm=1000.0, pcie=[10.0, 20.0], nvl=100.0)
    r0, r1 = rl["ranks"]
    assert r0["bytes"]["hbm"] == 600 * R + 1000 * R + 1000 * 16 + 1000 * 16 + 200 * R
    assert r0["bytes"]["nvlink_in"] == 300 * R and r0["bytes"]["nvlink_out"] == 200 * R
    assert r1["bytes"]["nvlink_out"] == 300 * R and r1["bytes"]["pcie"] == 300 * R
    assert abs(r0["t_s"]["pcie"] - 100 * R / 10e9) < 1e-15
    assert abs(r1["t_s"]["pcie"] - 300 * R / 20e9) < 1e-15
    assert r0["bound"] == "pcie" and r1["bound"] == "pcie"
    assert rl["bounding_rank"] == 1 and rl["t_roof_s"] == r1["t_roof_s"]
    # single pass: only queued peer keys pay the 16-B bucket round trip
    sp = bench.batch_roofline(P, n, R, kb, "single_pass", 1000.0, [10.0, 20.0], 100.0)
    assert sp["ranks"][0]["bytes"]["hbm"] == r0["bytes"]["hbm"] - 1000 * 16 + 300 * 16
    # split path: the timed kernel (K2) reads the bucket once and does no locate
    spl = bench.batch_roofline(P, n, R, kb, "split", 1000.0, [10.0, 20.0], 100.0)
    assert spl["ranks"][0]["kernel_bytes"]["hbm"] == 600 * R + 1000 * R + 8 * 1000 + 200 * R


def test_gpus_n_spawns_n_ranks_without_torchrun():
    """`python bench.py --gpus 2` outside torchrun re-launches itself with two ranks."""
    env = {k: v for k, v in os.environ.items() if k not in ("RANK", "WORLD_SIZE", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--print-world"],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr
    worlds = sorted(json.loads(l)["rank"] for l in r.stdout.splitlines() if l.startswith("{"))
    assert worlds == [0, 1]
    assert all(json.loads(l)["world_size"] == 2 for l in r.stdout.splitlines() if l.startswith("{"))


def test_world_size_mismatch_is_an_error():
    env = dict(os.environ, RANK="0", WORLD_SIZE="1", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "4", "--print-world"],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=300)
    assert r.returncode == 2 and "WORLD_SIZE" in r.stderr


def test_role_summary_groups_ctas_by_source():
    """bench.role_summary: rows [role, start, gather, role done, done] (ms) are grouped by
    source (this rank = local, num_gpus = host, other ids = peers), counted, and reported as
    [median, max] in us."""
    sys.path.insert(0, ROOT)
    import numpy as np
    import bench
    tl = np.array([[2, 0.0, 0.010, 0.100, 0.120],    # host (G = 2)
                   [2, 0.0, 0.012, 0.300, 0.310],
                   [1, 0.0, 0.011, 0.020, 0.200],    # peer 1
                   [0, 0.0, 0.010, 0.011, 0.150]],   # local (rank 0)
                  dtype=np.float32)
    r = bench.role_summary(tl, 2, 0)
    assert r["host"]["ctas"] == 2 and r["peer1"]["ctas"] == 1 and r["local"]["ctas"] == 1
    assert r["host"]["role_done"] == [200.0, 300.0]
    assert r["local"]["cta_done"] == [150.0, 150.0]
    assert r["peer1"]["gather_start"] == [11.0, 11.0]
