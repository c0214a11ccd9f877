O=gpurun_out/prof; mkdir -p $O
for v in "cfg2_S2bqp CFG2 2 2 1" "cfg2_S2bq CFG2 2 2 0" "g100_S2bqp G100 2 2 1" "g100_S2bq G100 2 2 0" "cfg2_S1bqp CFG2 1 2 1" "g100_S1bqp G100 1 2 1"; do
  set -- $v
  ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --cache-control none --clock-control none -k regex:nest_kernel -s 2 -c 1 --csv \
    python scripts/one_spmv.py --spec $2 --S $3 --mode spmd --U 1 --T 1024 --blocked 1 --vec $4 --persist $5 --iters 3 > $O/${1}_nocc.csv 2>&1
done
