# Round profile (run under gpurun): the launch list of the bench command, and one
# ncu --set full capture per (workload, configuration) the bench line reports --
# its roofline "traffic" comes from these (scripts/traffic_json.py).  Only the
# compact exports come back: raw csv pages + summaries.
O=gpurun_out/prof; mkdir -p $O
make host >/dev/null 2>&1
[ -z "$ONLY" ] && ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file $O/launches.csv \
    python bench.py --steps 20 --warmup 3 --no-cpu-baseline > $O/bench_under_ncu.log 2>&1
[ -z "$ONLY" ] && python scripts/launch_summary.py $O/launches.csv > $O/launches_summary.txt 2>&1
# tag spec S T blocked vec halo tps persist kernel-regex  (ONLY=<regex>: just the matching tags)
while read tag spec S T B V H TPS PS K; do
  [ -n "$ONLY" ] && ! [[ $tag =~ $ONLY ]] && continue
  ncu --set full --clock-control none --import-source on -k regex:$K -s 2 -c 1 -o /tmp/$tag -f \
      python scripts/one_spmv.py --spec $spec --S $S --mode spmd --U 1 --T $T --blocked $B --vec $V --halo $H \
      --tps $TPS --persist $PS --iters 3 > $O/$tag.log 2>&1
  ncu -i /tmp/$tag.ncu-rep --page raw --csv > $O/${tag}_raw.csv 2>/dev/null
  python scripts/ncu_summary.py /tmp/$tag.ncu-rep > $O/${tag}_summary.txt 2>&1
done <<'LIST'
cfg2_S2bqp CFG2 2 1024 1 2 0 0 1 nest_kernel
cfg2_S1bqp CFG2 1 1024 1 2 0 0 1 nest_kernel
g100_S2bqp G100 2 1024 1 2 0 0 1 nest_kernel
g100_S1bqp G100 1 1024 1 2 0 0 1 nest_kernel
cfg2_S2bq CFG2 2 1024 1 2 0 0 0 nest_kernel
cfg2_S2bv CFG2 2 1024 1 1 0 0 0 nest_kernel
cfg2_S1bv CFG2 1 1024 1 1 0 0 0 nest_kernel
g100_S2bq G100 2 1024 1 2 0 0 0 nest_kernel
g100_S2bv G100 2 1024 1 1 0 0 0 nest_kernel
g100_S1bv G100 1 1024 1 1 0 0 0 nest_kernel
cfg5_S8bv CFG5 8 1024 1 1 0 0 0 nest_kernel
cfg5_S1bv CFG5 1 1024 1 1 0 0 0 nest_kernel
cfg2_ring_S2v CFG2 2 768 0 1 4096 2 0 spmv_ring
LIST
[ -n "$ONLY" ] && exit 0
# per-instruction source pages of the headline and the S = 4 / 8 cfg2 kernels (wavefront attribution)
for v in "cfg2_S4bv 4" "cfg2_S8bv 8"; do
  set -- $v
  ncu --set full --clock-control none --import-source on -k regex:nest_kernel -s 2 -c 1 -o /tmp/$1 -f \
      python scripts/one_spmv.py --spec CFG2 --S $2 --mode spmd --U 1 --T 1024 --blocked 1 --vec 1 --iters 3 > $O/$1.log 2>&1
  ncu -i /tmp/$1.ncu-rep --page raw --csv > $O/${1}_raw.csv 2>/dev/null
  python scripts/ncu_summary.py /tmp/$1.ncu-rep > $O/${1}_summary.txt 2>&1
done
for t in cfg2_S2bq cfg2_S2bv cfg2_S4bv cfg2_S8bv; do
  ncu -i /tmp/$t.ncu-rep --page source --csv --print-source sass > $O/${t}_sass.csv 2>/dev/null
done
