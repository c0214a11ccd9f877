mkdir -p gpurun_out/prof
for v in "2 spmd 1 1024 4096" "4 spmd 1 1024 4096" "8 spmd 1 1024 4096"; do
  set -- $v
  ncu --set full --clock-control none --import-source on -k regex:spmv_staged -s 2 -c 1 \
      -o gpurun_out/prof/st3_S$1_$2_U$3_T$4_H$5 -f python scripts/one_spmv.py --S $1 --mode $2 --U $3 --T $4 --halo $5 --staged 1 --iters 3 > gpurun_out/prof/log3_S$1.txt 2>&1
done
