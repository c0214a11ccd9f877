mkdir -p gpurun_out/prof
ncu --set full --clock-control none --import-source on -k regex:spmv_xwin -s 2 -c 1 \
    -o gpurun_out/prof/xw2 -f python scripts/one_spmv.py --S 2 --mode spmd --U 1 --T 1024 --halo 4096 --iters 3 > gpurun_out/prof/log8.txt 2>&1
ncu -i gpurun_out/prof/xw2.ncu-rep --page source --csv --print-source sass > gpurun_out/prof/xw2_src.csv 2>/dev/null
