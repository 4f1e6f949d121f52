# A/B of an L2 persistence window over the BK (r02p2).  TB_BK_PERSIST was read only by the experimental build
# (run_br set cudaStreamAttributeAccessPolicyWindow around the br6 launch); that code was not kept, see
# profiles/r02p2_bk_l2_persist_ab.txt and DESIGN.md 7.1.
O=gpurun_out
for r in ${RATIOS:-0 0.5 1.0}; do
  if [ "$r" = "0" ]; then unset TB_BK_PERSIST; else export TB_BK_PERSIST=$r; fi
  timeout 400 python bench.py --no-sweep --no-cpu-baseline --steps 3 --warmup 3 > $O/r02p2_bench_$r.log 2>&1
  timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"br6_kernel|ks_kernel" -s 6 -c 2 --csv --log-file $O/r02p2_dram_$r.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-sweep > /dev/null 2>&1
done
