# A/B: alternate builds (scratch/lib_<name>.so) on one box; args: names...
G=${G:-16384}; L=${L:-2}; V=${V:-10}
for rep in 1 2; do for n in "$@"; do
  TB_LIB=scratch/lib_$n.so timeout 300 python bench.py --br-variant $V --lanes-per-cta $L --gates-per-gpu $G --steps 4 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$n', round(d['value']), round(d['roofline']['kernel_ms_per_launch'],2), d['clocks']['sm_mhz'])"
done; done
