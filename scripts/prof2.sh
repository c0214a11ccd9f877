mkdir -p gpurun_out/prof
for v in "8 spmd 4 1024 4096" "1 spmd 1 1024 4096"; do
  set -- $v
  ncu --set full --clock-control none --import-source on -k regex:spmv_xwin -s 2 -c 1 \
      -o gpurun_out/prof/xwin_S$1_$2_U$3_T$4 -f python scripts/one_spmv.py --S $1 --mode $2 --U $3 --T $4 --halo $5 --iters 3 > gpurun_out/prof/logx_S$1.txt 2>&1
done
ls -la gpurun_out/prof
