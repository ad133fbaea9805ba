# host-source experiments: probe (register flags) + library variants (bench --no-extra)
set -x
o=gpurun_out/probe3; mkdir -p $o
python tools/host_order_probe.py /tmp/rows.bin > $o/gen.txt
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/hop tools/host_order_probe.cu -lcuda
timeout 300 /tmp/hop /tmp/rows.bin 99900000 0 1 > $o/ro0.csv 2>&1
timeout 300 /tmp/hop /tmp/rows.bin 99900000 1 1 > $o/ro1.csv 2>&1
python __graft_entry__.py > /dev/null 2>&1
for hs in 12 24 48; do
 for hw in 8 16; do
  UGACHE_HOST_WARPS=$hw timeout 300 python bench.py --no-extra --no-verify --steps 10 --host-sms $hs > $o/b_${hs}_${hw}.json 2> $o/b_${hs}_${hw}.err
 done
done
