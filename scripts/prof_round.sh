# Round profile: launch list of the bench command + full capture of the dominant kernel.
set -x
mkdir -p gpurun_out/prof
ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/prof/launches.csv \
    python bench.py --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/prof/bench_under_ncu.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:nest_kernel -s 3 -c 1 \
    -o gpurun_out/prof/best -f python scripts/one_spmv.py --S 2 --mode spmd --U 1 --T 1024 --blocked 1 --iters 5 > gpurun_out/prof/best.log 2>&1
ncu -i gpurun_out/prof/best.ncu-rep --page raw --csv > gpurun_out/prof/best_raw.csv 2>/dev/null
