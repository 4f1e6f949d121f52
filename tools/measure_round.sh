#!/bin/bash
# Round measurement batch on one B200 (run under gpurun from the repo root):
#   bench line (default command), reference arm, BR-kernel DRAM traffic at the bench size, launch list of the
#   default command, and every BASELINE config (tools/workloads.py).  Outputs: gpurun_out/${TAG}_*.
TAG=${TAG:-r01}
O=gpurun_out
python bench.py > $O/${TAG}_bench.log 2>&1; tail -1 $O/${TAG}_bench.log > $O/${TAG}_bench.json
python bench.py --impl reference > $O/${TAG}_ref.log 2>&1; tail -1 $O/${TAG}_ref.log > $O/${TAG}_ref.json
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum \
    --clock-control none -k regex:br6_kernel -s 3 -c 1 --csv --log-file $O/${TAG}_br6_dram.csv \
    python bench.py --steps 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/${TAG}_launches.csv \
    python bench.py --no-cpu-baseline --steps 2 --warmup 3 > /dev/null 2>&1
[ -n "$NO_WORKLOADS" ] || python tools/workloads.py > $O/${TAG}_workloads.jsonl 2> $O/${TAG}_workloads.err
echo done
