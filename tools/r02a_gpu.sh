#!/bin/bash
# Round-2 first GPU batch: full GPU suite (incl. full-size parity), smoke, default bench, the N > 1 bench path on
# one GPU (--one-gpu-ranks), the loud failure of --gpus 8 on a one-GPU node, ncu of the shipped key switch.
O=gpurun_out
T=${TAG:-r02a}
timeout 2400 python -m pytest tests -m gpu -x -q > $O/${T}_gpu_tests.log 2>&1; echo "pytest exit $?" >> $O/${T}_gpu_tests.log
timeout 300 python __graft_entry__.py smoke > $O/${T}_smoke.log 2>&1; echo "smoke exit $?" >> $O/${T}_smoke.log
timeout 600 python bench.py > $O/${T}_bench.log 2>&1; tail -1 $O/${T}_bench.log > $O/${T}_bench.json
timeout 600 python bench.py --gpus 2 --one-gpu-ranks --gates-per-gpu 4096 --steps 2 --warmup 3 > $O/${T}_bench_n2.log 2>&1
echo "n2 exit $?" >> $O/${T}_bench_n2.log
timeout 120 python bench.py --gpus 8 > $O/${T}_bench_n8.log 2>&1; echo "n8 exit $?" >> $O/${T}_bench_n8.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ks_kernel -s 3 -c 1 \
    -o $O/${T}_ncu_ks python bench.py --steps 1 --no-cpu-baseline --no-e2e > $O/${T}_ncu_ks.log 2>&1
echo done
