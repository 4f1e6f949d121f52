#!/bin/bash
O=gpurun_out
T=${TAG:-r02p}
timeout 1200 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_workloads.py -x -q > $O/${T}_tests.log 2>&1; echo "exit $?" >> $O/${T}_tests.log
timeout 900 python tools/e2e_overlap.py > $O/${T}_e2e_overlap.jsonl 2> $O/${T}_e2e_overlap.err
echo done
