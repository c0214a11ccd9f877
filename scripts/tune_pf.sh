for r in 0 1 2 3 4 6; do
  echo "rounds=$r"; NEST_L2PF_ROUNDS=$r timeout 120 python scripts/sweep_spmv.py --iters 5 --simdlens 1,2,4 --modes spmd --unrolls 1 --hints 0 --threads 512,1024 --halos 0 --staged 0 --blocked 1 2>&1 | grep "^{" | sed 's/"hints": 0, "halo": 0, "staged": 0, //; s/, "min_ms.*//'
done
