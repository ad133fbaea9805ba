set -x
o=gpurun_out/r1i; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o /tmp/hgp tools/hbm_gather_probe.cu
timeout 300 /tmp/hgp 57 500000 512 > $o/hbm_gather_512.csv 2>&1
timeout 300 /tmp/hgp 57 500000 1536 > $o/hbm_gather_1536.csv 2>&1
for lb in 0 1; do for c in 0.1 1.0; do
  UGACHE_LOCAL_BULK=$lb timeout 600 python bench.py --cache-ratio $c --no-verify --e2e-steps 1 --cpu-seconds 1 --no-extra > $o/bench_c${c}_lb$lb.json 2> $o/bench_c${c}_lb$lb.err
done; done
