#!/bin/bash
# Build a libbmr variant with extra -D flags into variants/libbmr_<name>.so (sweeps: BMR_LIB=...).
# usage: tools/build_variant.sh NAME "-DFOO=1 -DBAR=2"
set -e
name=$1; defs=$2
mkdir -p build/var_$name variants
NCCL_INC=$(python3 -c "import nvidia.nccl, os; print(os.path.join(list(nvidia.nccl.__path__)[0], 'include'))" 2>/dev/null || echo /usr/include)
NVFLAGS="-O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC --expt-relaxed-constexpr -ftz=false -prec-div=true -prec-sqrt=true"
objs=""
pids=""
for f in paper_conf_ipps_jim11_b200/csrc/*.cu; do
  b=$(basename $f .cu)
  nvcc $NVFLAGS $defs -Iinclude -I$NCCL_INC -c -o build/var_$name/$b.o $f &
  pids="$pids $!"
  objs="$objs build/var_$name/$b.o"
done
for p in $pids; do wait $p; done
nvcc -gencode arch=compute_100a,code=sm_100a -shared --cudart static -o variants/libbmr_$name.so $objs -ldl
echo variants/libbmr_$name.so
