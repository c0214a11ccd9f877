# ncu --set full of one x-ring SpMV launch on cfg2 + its source page (developer profiling)
O=gpurun_out/prof_ring; mkdir -p $O
make host >/dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:spmv_ring -s 1 -c 1 -o /tmp/ring -f python scripts/one_spmv.py --spec CFG2 --S 2 --T 768 --vec 2 --halo 4096 --tps 2 --iters 2 > $O/ring.log 2>&1
ncu -i /tmp/ring.ncu-rep --page source --csv --print-source sass > $O/ring_sass.csv 2>/dev/null
python scripts/ncu_summary.py /tmp/ring.ncu-rep > $O/ring_summary.txt 2>&1
