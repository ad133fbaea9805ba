set -x
o=gpurun_out/r1h; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 300 python -m pytest tests -m gpu -x -q -k "row_sizes or fused or single_gpu or fake_peer" > $o/pytest_bulk.txt 2>&1
tail -3 $o/pytest_bulk.txt
timeout 900 python -m pytest tests -m gpu -x -q > $o/pytest_all.txt 2>&1
tail -3 $o/pytest_all.txt
for c in 1.0 0.1; do
  timeout 600 python bench.py --cache-ratio $c --no-verify --e2e-steps 1 --cpu-seconds 1 > $o/bench_c$c.json 2> $o/bench_c$c.err
done
