#!/bin/bash
# throwaway tuning sweep: variant x lanes-per-CTA at 16384 gates
for V in 6 2; do for L in 1 2 3 4; do
  TB_BR_VARIANT=$V timeout 200 python bench.py --gates-per-gpu ${G:-16384} --lanes-per-cta $L --steps 3 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('V=$V L=$L', round(d['value']), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], round(d['latency_ms']['level_of_1_gate'],2), round(d['roofline']['ks_kernel_ms_per_launch'],2))"
done; done
