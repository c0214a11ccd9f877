mkdir -p gpurun_out/prof
ncu --set full --clock-control none --import-source on -k regex:spmv_staged -s 2 -c 1 \
    -o gpurun_out/prof/st5_S8_T512_H4096 -f python scripts/one_spmv.py --S 8 --mode spmd --U 1 --T 512 --halo 4096 --staged 1 --iters 3 > gpurun_out/prof/log5.txt 2>&1
ncu -i gpurun_out/prof/st5_S8_T512_H4096.ncu-rep --page source --csv --print-source sass > gpurun_out/prof/st5_src.csv 2>/dev/null
