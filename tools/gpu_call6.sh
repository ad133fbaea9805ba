set -x
o=gpurun_out/r1f; mkdir -p $o
python __graft_entry__.py > $o/build.txt 2>&1
timeout 600 python -m pytest tests -m gpu -x -q -k "message or fused or single_gpu" > $o/pytest_msg.txt 2>&1
timeout 900 python tools/message_compare.py --out $o/message_compare.json > $o/message_compare.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $o/launches.csv python bench.py --steps 3 --warmup 3 --no-extra --no-verify > $o/ncu_launch_bench.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:fused_extract -s 5 -c 1 -o $o/prof_fused python bench.py --steps 2 --warmup 3 --no-extra --no-verify --no-host-tier > $o/ncu_full.log 2>&1
