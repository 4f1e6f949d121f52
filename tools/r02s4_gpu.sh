O=gpurun_out
T=r02s4
timeout 900 python tools/latency.py 0 11 16 > $O/${T}_latency.jsonl 2> $O/${T}_latency.err
timeout 900 python bench.py > $O/${T}_bench.log 2>&1; tail -1 $O/${T}_bench.log > $O/${T}_bench.json
timeout 1200 python tools/workloads.py --only cfg1 > $O/${T}_cfg1.jsonl 2>&1
timeout 1200 python tools/workloads.py --only cfg2 > $O/${T}_cfg2.jsonl 2>&1
timeout 1200 python tools/workloads.py --only cfg4 > $O/${T}_cfg4.jsonl 2>&1
echo done
