# L1 / shared carve-out experiment on the headline SpMV (NEST_CARVEOUT, percent of max shared).
mkdir -p gpurun_out/carve
for c in default 0 25 100; do
  if [ $c = default ]; then unset NEST_CARVEOUT; else export NEST_CARVEOUT=$c; fi
  timeout 300 python bench.py --no-cpu-baseline --steps 100 > gpurun_out/carve/bench_$c.log 2>&1
  timeout 300 ncu --metrics gpu__time_duration.sum,l1tex__t_sector_hit_rate.pct,launch__shared_mem_config_size,dram__bytes_read.sum,l1tex__throughput.avg.pct_of_peak_sustained_active \
      --clock-control none -k regex:nest_kernel -s 2 -c 1 --csv \
      python scripts/one_spmv.py --S 2 --mode spmd --U 1 --T 1024 --blocked 1 --vec 1 --iters 4 > gpurun_out/carve/ncu_$c.csv 2>&1
done
unset NEST_CARVEOUT
