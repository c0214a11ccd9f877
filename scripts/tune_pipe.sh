for pipe in 0 1; do
  echo "pipe=$pipe"; NEST_RP_PIPE=$pipe timeout 120 python scripts/sweep_spmv.py --iters 5 --simdlens 1,2,4 --modes spmd,generic_smem --unrolls 1,2 --hints 0 --threads 512,1024 --halos 0 --staged 0 --blocked 1 2>&1 | grep "^{" | sed 's/"hints": 0, "halo": 0, "staged": 0, //; s/, "min_ms.*//'
done
