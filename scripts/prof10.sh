mkdir -p gpurun_out/prof
ncu --set full --clock-control none --import-source on -k regex:nest_kernel -s 3 -c 1 \
    -o /tmp/p10 -f python scripts/one_spmv.py --S 2 --mode spmd --U 1 --T 1024 --blocked 1 --vec 1 --iters 5 > gpurun_out/prof/p10.log 2>&1
ncu -i /tmp/p10.ncu-rep --page source --csv --print-source sass > gpurun_out/prof/p10_src.csv 2>/dev/null
