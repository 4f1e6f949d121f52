#!/bin/bash
# Mixed-variant sweep (br6 + brf co-resident): bench line per configuration, one box.
# usage: tools/mix_sweep.sh "V MIX" ...   e.g. "6 -" "12 300,118784,1"
G=${G:-65536}
for cfg in "$@"; do
  set -- $cfg; V=$1; MIX=${2:-300,118784,1}
  timeout 300 python bench.py --br-variant $V --mix $MIX --gates-per-gpu $G --steps ${K:-3} --warmup 3 \
      --no-cpu-baseline --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$V $MIX', round(d['value']), round(d['roofline']['kernel_ms_per_launch'],2), d['clocks']['sm_mhz'])" || echo "$V $MIX failed"
done
