# N = 2 bench path on one B200 (two ranks share the device: gloo control plane, real cudaIpc peers).
set -x
o=gpurun_out/r2c; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
T="timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1"
$T --master-port 29511 bench.py --gpus 2 --workload tiny --steps 10 --warmup 3 > $o/tiny_n2.json 2> $o/tiny_n2.err
$T --master-port 29512 bench.py --impl reference --gpus 2 --workload tiny --steps 3 --warmup 3 > $o/tiny_n2_ref.json 2> $o/tiny_n2_ref.err
$T --master-port 29513 bench.py --gpus 2 --cache-ratio 0.1 --workload gnn_pa@0.25 --steps 10 --warmup 3 --cpu-seconds 1 --e2e-steps 2 > $o/pa25_n2.json 2> $o/pa25_n2.err
