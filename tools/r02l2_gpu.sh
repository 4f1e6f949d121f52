#!/bin/bash
# brl2 (2-SM FP64 latency kernel) batch: latency-mode tests, latency table, cfg4 workloads, sanitizers on brl2
O=gpurun_out
T=${TAG:-r02l2}
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tc.py -x -q -k "latency_mode or domains" > $O/${T}_tests.log 2>&1; echo "exit $?" >> $O/${T}_tests.log
timeout 900 python tools/latency.py 0 16 6 > $O/${T}_latency.jsonl 2> $O/${T}_latency.err
timeout 1200 python tools/workloads.py --only cfg4 > $O/${T}_cfg4.jsonl 2>&1
timeout 1200 python tools/workloads.py --only cfg2 > $O/${T}_cfg2.jsonl 2>&1
for tool in memcheck synccheck racecheck; do
  TB_SAN_LATENCY=1 timeout 1200 compute-sanitizer --tool $tool python tools/sanitize_run.py > $O/${T}_sanitize_lat_$tool.log 2>&1
done
echo done
