#!/bin/bash
# Round-2 session-2 final batch (one B200): full GPU suite, smoke, latency table, bench line, reference arm,
# BR DRAM traffic at the bench size, launch list of the default command, every BASELINE config.
# (compute-sanitizer is closed on this GPU pool since round 2 session 2: not run.)
O=gpurun_out
T=${TAG:-r02s2}
timeout 1800 python -m pytest tests -m gpu -q > $O/${T}_gpu_tests.log 2>&1; echo "exit $?" >> $O/${T}_gpu_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/${T}_smoke.log 2>&1; echo "exit $?" >> $O/${T}_smoke.log
timeout 900 python tools/latency.py 0 11 16 > $O/${T}_latency.jsonl 2> $O/${T}_latency.err
timeout 900 python bench.py > $O/${T}_bench.log 2>&1; tail -1 $O/${T}_bench.log > $O/${T}_bench.json
timeout 600 python bench.py --impl reference > $O/${T}_ref.log 2>&1; tail -1 $O/${T}_ref.log > $O/${T}_ref.json
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum \
    --clock-control none -k regex:br6_kernel -s 3 -c 1 --csv --log-file $O/${T}_br6_dram.csv \
    python bench.py --steps 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/${T}_launches.csv \
    python bench.py --no-cpu-baseline --steps 2 --warmup 3 > /dev/null 2>&1
timeout 1500 python tools/workloads.py > $O/${T}_workloads.jsonl 2> $O/${T}_workloads.err
echo done
