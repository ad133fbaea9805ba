set -x
o=gpurun_out/probe5; mkdir -p $o
for b in 0 1 2 3; do python tools/host_order_probe.py /tmp/rows$b.bin gnn_pa 0.1 $b >> $o/gen.txt; done
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/hop tools/host_order_probe.cu -lcuda
R=/tmp/rows0.bin,/tmp/rows1.bin,/tmp/rows2.bin,/tmp/rows3.bin
timeout 600 /tmp/hop $R 99900000 0 0 0 > $o/m0_full.csv 2>&1
for m in 1 2 3; do timeout 600 /tmp/hop $R 99900000 0 1 $m > $o/m$m.csv 2>&1; done
echo 25000 > /proc/sys/vm/nr_hugepages; cat /proc/sys/vm/nr_hugepages > $o/hugetlb.txt
timeout 600 /tmp/hop $R 99900000 0 1 4 > $o/m4.csv 2>&1
echo 0 > /proc/sys/vm/nr_hugepages
