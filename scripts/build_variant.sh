#!/bin/bash
# Build a variant of libnest.so with extra nvcc defines into build_<name>/ (A/B
# experiments on the GPU box: copy it over paper_conf_icpp_wrightdtcc23_b200/libnest.so).
# Only the SpMV tuple-body translation units are recompiled; the rest come from build/.
# usage: scripts/build_variant.sh h0 -DNEST_VEC_HEAD=0   (VARIANT_ALL=1: recompile every unit)
set -e
name=$1; shift
cd "$(dirname "$0")/.."
NCCL=$(python -c "import nvidia.nccl,os;print(list(nvidia.nccl.__path__)[0])")
FL="-O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC -Xcompiler -fvisibility=hidden -Iinclude -Ipaper_conf_icpp_wrightdtcc23_b200/csrc -I$NCCL/include --expt-relaxed-constexpr"
mkdir -p build_$name
for f in paper_conf_icpp_wrightdtcc23_b200/csrc/*.cu; do
  b=$(basename $f .cu)
  if [ -n "$VARIANT_ALL" ] || grep -q "SpmvVecBody\|BatchedVecBody\|StencilBody\|LaplaceVecBody" $f || [ $b = spmv_vec2 ] || [ $b = spmv_vec4 ]; then
    nvcc $FL "$@" -c $f -o build_$name/$b.o &
  else
    cp build/$b.o build_$name/$b.o
  fi
done
wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -L$NCCL/lib -l:libnccl.so.2 \
     -Xlinker -rpath,$NCCL/lib -o build_$name/libnest.so build_$name/*.o
echo built build_$name/libnest.so
rm -f build_$name/*.o   # only the library travels to the GPU box
