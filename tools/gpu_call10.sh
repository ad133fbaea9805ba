set -x
o=gpurun_out/r1j; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 300 python -m pytest tests -m gpu -x -q -k "row_sizes or fused" > $o/pytest.txt 2>&1; tail -2 $o/pytest.txt
for rep in 1 2; do for lb in 0 1; do for c in 0.1 1.0; do
  UGACHE_LOCAL_BULK=$lb timeout 600 python bench.py --cache-ratio $c --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra > $o/bench_c${c}_lb${lb}_$rep.json 2> $o/bench_c${c}_lb${lb}_$rep.err
done; done; done
