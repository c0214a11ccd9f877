for cfg in "4 1 512" "4 2 1024" "2 1 1024" "8 2 1024" "4 1 1024"; do
 set -- $cfg
 for ns in 3; do for r in 256; do
  NEST_DEBUG_PLAN=1 NEST_STAGED_NS=$ns NEST_STAGED_R=$r timeout 120 python scripts/sweep_spmv.py --iters 3 --simdlens $1 --modes spmd --unrolls $2 --hints 0 --threads $3 --halos 4096 --staged 1 2>&1 | grep -E "staged plan|^\{" | tail -2 | tr '\n' ' ' | sed 's/"hints": 0, //; s/"staged": 1, //; s/"min_ms.*//'; echo
 done; done
done
