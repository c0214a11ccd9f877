mkdir -p gpurun_out/prof
NEST_STAGED_NS=3 NEST_STAGED_R=256 ncu --set full --clock-control none --import-source on -k regex:spmv_staged -s 2 -c 1 \
    -o gpurun_out/prof/st6 -f python scripts/one_spmv.py --S 4 --mode spmd --U 1 --T 512 --halo 4096 --staged 1 --iters 3 > gpurun_out/prof/log6.txt 2>&1
ncu -i gpurun_out/prof/st6.ncu-rep --page source --csv --print-source sass > gpurun_out/prof/st6_src.csv 2>/dev/null
