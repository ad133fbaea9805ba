set -x
o=gpurun_out/r1k; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 300 python -m pytest tests -m gpu -x -q -k "row_sizes or fused or timing" > $o/pytest.txt 2>&1; tail -2 $o/pytest.txt
for lb in 0 3 2; do for c in 0.1 1.0; do
  UGACHE_LOCAL_BULK=$lb timeout 600 python bench.py --cache-ratio $c --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra > $o/bench_c${c}_lb${lb}.json 2> $o/bench_c${c}_lb${lb}.err
done; done
timeout 600 python bench.py --workload gnn_mag@0.15 --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra > $o/bench_mag.json 2> $o/bench_mag.err
timeout 600 python bench.py --workload dlr_criteo@0.15 --no-verify --e2e-steps 1 --cpu-seconds 1 > $o/bench_dlr.json 2> $o/bench_dlr.err
timeout 600 python bench.py --workload dlr_criteo@0.15 --cache-ratio 0.02 --no-verify --e2e-steps 1 --cpu-seconds 1 > $o/bench_dlr2.json 2> $o/bench_dlr2.err
