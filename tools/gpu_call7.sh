set -x
o=gpurun_out/r1g; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:fused_extract -s 3 -c 1 -o $o/prof_fused python bench.py --steps 2 --warmup 3 --no-extra --no-verify --no-host-tier --e2e-steps 1 --cpu-seconds 0.5 > $o/ncu_full.log 2>&1
for c in 1.0 0.3; do
  timeout 600 python bench.py --cache-ratio $c --no-verify --e2e-steps 1 --cpu-seconds 1 > $o/bench_c$c.json 2> $o/bench_c$c.err
done
timeout 600 python bench.py --workload gnn_pa --cache-ratio 1.0 --steps 20 --no-verify --e2e-steps 1 --cpu-seconds 1 --policy replication > $o/bench_c1_rep.json 2> $o/bench_c1_rep.err
