#!/bin/bash
O=gpurun_out
T=${TAG:-r02v}
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "latency_mode" > $O/${T}_lat_tests.log 2>&1; echo "exit $?" >> $O/${T}_lat_tests.log
timeout 600 python tools/latency.py 13 11 9 > $O/${T}_latency.jsonl 2> $O/${T}_latency.err
echo done
