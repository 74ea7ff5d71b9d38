#!/usr/bin/env bash
# build/<name>/libpccheck.so with extra nvcc flags for kernels.cu (A/B experiments; PCC_LIB=... to load)
set -eu
name=$1; shift
NCCL_DIR=$(python -c "import nvidia.nccl, os; print(os.path.dirname(nvidia.nccl.__path__[0]) + '/nccl')")
mkdir -p build/$name
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-fvisibility=hidden -Xptxas -v \
  -I$NCCL_DIR/include "$@" -c paper_conf_asplos_strati0k25_b200/csrc/kernels.cu -o build/$name/kernels.o 2> build/$name/ptxas.log
for f in runtime commit kapi host_api; do
  g++ -O2 -fPIC -std=c++17 -msse4.2 -I/usr/local/cuda/include -I$NCCL_DIR/include -DPCC_NCCL_LIBDIR=\"$NCCL_DIR/lib\" \
      -fvisibility=hidden "$@" -c paper_conf_asplos_strati0k25_b200/csrc/$f.cpp -o build/$name/$f.o
done
g++ -shared -o build/$name/libpccheck.so build/$name/*.o -L/usr/local/cuda/lib64 -lcudart_static -ldl -lpthread -lrt -Wl,--exclude-libs,ALL
grep -A1 "k_snap_tmaILb1" build/$name/ptxas.log | grep -oE "Used [0-9]+ registers|[0-9]+ bytes spill stores" | tr '\n' ' '; echo " <- $name $*"
