set -x
mkdir -p gpurun_out/prof
for v in "1 spmd 1" "4 spmd 1" "8 spmd 1" "8 generic_smem 1"; do
  set -- $v
  ncu --set full --clock-control none --import-source on -k regex:nest_kernel -s 2 -c 1 \
      -o gpurun_out/prof/spmv_S$1_$2_U$3 -f python scripts/one_spmv.py --S $1 --mode $2 --U $3 --iters 3 > gpurun_out/prof/log_S$1_$2.txt 2>&1
done
ls -la gpurun_out/prof
