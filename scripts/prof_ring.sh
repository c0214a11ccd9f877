# ncu --set full of one x-ring SpMV launch on cfg2 (developer profiling)
make host >/dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:spmv_ring -s 1 -c 1 -o gpurun_out/ring_s2_tps1 python scripts/one_spmv.py --spec CFG2 --S 2 --T 1024 --vec 1 --halo 4096 --tps 1 --iters 2 > gpurun_out/prof_ring.log 2>&1
python scripts/ncu_summary.py gpurun_out/ring_s2_tps1.ncu-rep > gpurun_out/prof_ring_summary.txt 2>&1
