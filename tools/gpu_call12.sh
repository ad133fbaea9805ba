set -x
o=gpurun_out/r1m; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $o/pytest.txt 2>&1; tail -2 $o/pytest.txt
for ew in 0 1; do
  UGACHE_EARLY_WALK=$ew timeout 600 python bench.py --workload dlr_criteo@0.15 --no-verify --e2e-steps 1 --cpu-seconds 1 > $o/dlr_ew$ew.json 2> $o/dlr_ew$ew.err
  UGACHE_EARLY_WALK=$ew timeout 600 python bench.py --workload dlr_criteo@0.15 --cache-ratio 0.02 --no-verify --e2e-steps 1 --cpu-seconds 1 > $o/dlr2_ew$ew.json 2> $o/dlr2_ew$ew.err
  UGACHE_EARLY_WALK=$ew timeout 600 python bench.py --no-verify --e2e-steps 1 --cpu-seconds 1 > $o/pa_ew$ew.json 2> $o/pa_ew$ew.err
done
