# Dense-host threshold check: ordered two-phase (auto) vs forced single pass, gnn_pa c = 0.1-0.5.
set -x
o=gpurun_out/r2b; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
for c in 0.1 0.2 0.3 0.5; do
  timeout 600 python bench.py --cache-ratio $c --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra > $o/pa_c${c}_auto.json 2> $o/pa_c${c}_auto.err
  UGACHE_HOST_SORT_MIN=1000000000 timeout 600 python bench.py --cache-ratio $c --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra > $o/pa_c${c}_sp.json 2> $o/pa_c${c}_sp.err
done
