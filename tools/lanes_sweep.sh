mkdir -p gpurun_out
for G in 592 1024 1536 2048; do for L in 1 2 3 4; do
  timeout 200 python bench.py --gates-per-gpu $G --lanes-per-cta $L --steps 5 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('G=$G L=$L', round(d['value']), round(d['ms_per_step'],2), round(d['roofline']['kernel_ms_per_launch'],2), round(d['roofline']['ks_kernel_ms_per_launch'],2), d['clocks']['sm_mhz'])" >> gpurun_out/r01f_lanes_sweep.txt
done; done
