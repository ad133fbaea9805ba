set -x
o=gpurun_out/probe4; mkdir -p $o
for b in 0 1 2 3; do python tools/host_order_probe.py /tmp/rows$b.bin gnn_pa 0.1 $b >> $o/gen.txt; done
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/hop tools/host_order_probe.cu -lcuda
cat /sys/kernel/mm/transparent_hugepage/enabled > $o/thp.txt
timeout 600 /tmp/hop /tmp/rows0.bin,/tmp/rows1.bin,/tmp/rows2.bin,/tmp/rows3.bin 99900000 0 1 > $o/multi.csv 2>&1
timeout 600 /tmp/hop /tmp/rows0.bin 99900000 0 1 > $o/single.csv 2>&1
grep -i huge /proc/meminfo >> $o/thp.txt
