#!/bin/bash
O=gpurun_out
T=${TAG:-r02y}
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tc.py -x -q -k "latency_mode or domains or variants" > $O/${T}_tests.log 2>&1; echo "exit $?" >> $O/${T}_tests.log
timeout 600 python tools/latency.py 0 13 11 9 > $O/${T}_latency.jsonl 2> $O/${T}_latency.err
timeout 1200 python tools/workloads.py --only cfg4 > $O/${T}_cfg4.jsonl 2>&1
echo done
