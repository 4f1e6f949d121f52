#!/bin/bash
# Round-2 measurement batch (one B200): bench line (default), reference arm, BR-kernel DRAM traffic at the bench
# size, launch list of the default command, every BASELINE config, sanitizers over the current kernel set.
O=gpurun_out
T=${TAG:-r02r}
timeout 900 python bench.py > $O/${T}_bench.log 2>&1; tail -1 $O/${T}_bench.log > $O/${T}_bench.json
timeout 600 python bench.py --impl reference > $O/${T}_ref.log 2>&1; tail -1 $O/${T}_ref.log > $O/${T}_ref.json
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum \
    --clock-control none -k regex:br6_kernel -s 3 -c 1 --csv --log-file $O/${T}_br6_dram.csv \
    python bench.py --steps 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/${T}_launches.csv \
    python bench.py --no-cpu-baseline --steps 2 --warmup 3 > /dev/null 2>&1
timeout 1200 python tools/workloads.py > $O/${T}_workloads.jsonl 2> $O/${T}_workloads.err
for tool in memcheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool python tools/sanitize_run.py > $O/${T}_sanitize_$tool.log 2>&1
done
TB_SAN_QUICK=1 timeout 1200 compute-sanitizer --tool racecheck python tools/sanitize_run.py > $O/${T}_sanitize_racecheck.log 2>&1
TB_SAN_BRT=1 timeout 1800 compute-sanitizer --tool racecheck python tools/sanitize_run.py > $O/${T}_sanitize_racecheck_brt.log 2>&1
echo done
