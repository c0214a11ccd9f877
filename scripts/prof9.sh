mkdir -p gpurun_out/prof
ncu --set full --clock-control none --import-source on -k regex:nest_kernel -s 3 -c 1 \
    -o gpurun_out/prof/vec_S1 -f python scripts/one_spmv.py --S 1 --mode spmd --U 1 --T 1024 --blocked 1 --vec 1 --iters 5 > gpurun_out/prof/log9.txt 2>&1
ncu -i gpurun_out/prof/vec_S1.ncu-rep --page raw --csv > gpurun_out/prof/vec_S1_raw.csv 2>/dev/null
ncu -i gpurun_out/prof/vec_S1.ncu-rep --page source --csv --print-source sass > gpurun_out/prof/vec_S1_src.csv 2>/dev/null
