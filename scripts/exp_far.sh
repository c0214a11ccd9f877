#!/bin/bash
# DRAM traffic of the headline SpMV kernel vs the fraction of far (uniformly random) columns.
O=gpurun_out/exp_far; mkdir -p $O
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum
for fd in 1073741824 64 16 4; do
  ncu --metrics $M --clock-control none -k regex:nest_kernel -s 2 -c 1 --csv python scripts/one_spmv.py --S 2 --T 1024 --blocked 1 --vec 1 --far_den $fd --iters 3 > $O/ncu_fd$fd.csv 2>&1
done
ncu --metrics $M --clock-control none -k regex:nest_kernel -s 2 -c 1 --csv python scripts/one_spmv.py --spec CFG2_UNIFORM --S 2 --T 1024 --blocked 1 --vec 1 --iters 3 > $O/ncu_uniform.csv 2>&1
