#!/bin/bash
# A/B of the auto lanes-per-CTA choice: GPU suite, bench at the bench size and mid sizes, workloads.
O=gpurun_out; T=${TAG:-r01g}
python -m pytest tests -m gpu -x -q > $O/${T}_gpu_tests.log 2>&1
for G in 1024 1536 2048; do
  timeout 200 python bench.py --gates-per-gpu $G --steps 5 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 >> $O/${T}_mid.jsonl
done
python bench.py > $O/${T}_bench.log 2>&1; tail -1 $O/${T}_bench.log > $O/${T}_bench.json
python tools/workloads.py > $O/${T}_workloads.jsonl 2> $O/${T}_workloads.err
echo done
