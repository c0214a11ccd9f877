mkdir -p gpurun_out/prof
for S in 2 4; do
ncu --set full --clock-control none --import-source on -k regex:nest_kernel -s 2 -c 1 \
    -o gpurun_out/prof/blk_S$S -f python scripts/one_spmv.py --S $S --mode spmd --U 1 --T 1024 --blocked 1 --iters 3 > gpurun_out/prof/log7.txt 2>&1
done
ncu -i gpurun_out/prof/blk_S2.ncu-rep --page source --csv --print-source sass > gpurun_out/prof/blk_S2_src.csv 2>/dev/null
