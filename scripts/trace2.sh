for cfg in "4 1 512 256" "4 1 1024 256" "2 1 1024 512"; do
 set -- $cfg
 NEST_DEBUG_PLAN=1 NEST_TRACE=1 NEST_STAGED_NS=3 NEST_STAGED_R=$4 python scripts/one_spmv.py --S $1 --mode spmd --U $2 --T $3 --halo 4096 --staged 1 --iters 1 > gpurun_out/trace_$1_$3.txt 2>&1
 grep plan gpurun_out/trace_$1_$3.txt; grep "trace\] [345][0-9] " gpurun_out/trace_$1_$3.txt | head -8
done
