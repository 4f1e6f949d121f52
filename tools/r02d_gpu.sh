#!/bin/bash
O=gpurun_out
T=${TAG:-r02d}
timeout 180 python -m pytest tests/test_gpu_tc.py -x -q > $O/${T}_tc.log 2>&1; rc=$?; echo "exit $rc" >> $O/${T}_tc.log
[ $rc -eq 0 ] || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "variants_bit_exact" > $O/${T}_var.log 2>&1; rc=$?; echo "exit $rc" >> $O/${T}_var.log
[ $rc -eq 0 ] || exit 1
timeout 300 python bench.py --br-variant 12 --steps 3 --no-cpu-baseline --no-e2e > $O/${T}_bench12.log 2>&1
tail -1 $O/${T}_bench12.log > $O/${T}_bench12.json
echo done
