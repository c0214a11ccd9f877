# Round profile: launch list of the bench command + full capture of the headline kernel
# (only the compact exports come back: raw csv + summaries).
mkdir -p gpurun_out/prof
ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/prof/launches.csv \
    python bench.py --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/prof/bench_under_ncu.log 2>&1
for v in "2 best" "1 s1"; do
  set -- $v
  ncu --set full --clock-control none --import-source on -k regex:nest_kernel -s 3 -c 1 \
      -o /tmp/$2 -f python scripts/one_spmv.py --S $1 --mode spmd --U 1 --T 1024 --blocked 1 --vec 1 --iters 5 > gpurun_out/prof/$2.log 2>&1
  ncu -i /tmp/$2.ncu-rep --page raw --csv > gpurun_out/prof/$2_raw.csv 2>/dev/null
  python scripts/ncu_summary.py /tmp/$2.ncu-rep > gpurun_out/prof/$2_summary.txt 2>&1
done
python scripts/launch_summary.py gpurun_out/prof/launches.csv > gpurun_out/prof/launches_summary.txt 2>&1
