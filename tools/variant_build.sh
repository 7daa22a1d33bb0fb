#!/bin/bash
# Build an experimental libsj variant (k=8 kernels for dims 2/3/6 only: -DSJ_QUICK) into
# exp/libsj_<name>.so; run it with SJ_LIB_PATH=exp/libsj_<name>.so.  usage: variant_build.sh name [nvcc flags]
set -e
name=$1; shift
cd "$(dirname "$0")/../paper_conf_ipps_galletg19_b200/csrc"
B=/tmp/x/vb_$name; mkdir -p $B ../../exp
FL="-DSJ_QUICK $* -O3 -gencode arch=compute_100a,code=sm_100a -lineinfo -std=c++17 --fmad=false -Xcompiler -fPIC -ccbin /usr/bin/g++"
for f in primitives grid_build join_kernel sj_runtime diag; do
  /usr/local/cuda/bin/nvcc $FL -c $f.cu -o $B/$f.o &
done
wait
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o ../../exp/libsj_$name.so $B/*.o
echo built exp/libsj_$name.so
