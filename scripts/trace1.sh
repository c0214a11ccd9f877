NEST_DEBUG_PLAN=1 NEST_TRACE=1 NEST_STAGED_NS=4 NEST_STAGED_R=256 python scripts/one_spmv.py --S 8 --mode spmd --U 1 --T 512 --halo 4096 --staged 1 --iters 1 > gpurun_out/trace1.txt 2>&1
