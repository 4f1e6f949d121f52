#!/bin/bash
# latency A/B of alternative builds (scratch/lib_<name>.so) for one narrow kernel K (default 13): one-gate level
K=${K:-13}
for n in "$@"; do
  TB_LIB=scratch/lib_$n.so timeout 300 python tools/latency.py $K 2>/dev/null | python -c "import json,sys; r=[json.loads(l) for l in sys.stdin]; print('$n', [(d['lanes'], round(d['level_ms'],3)) for d in r])"
done
