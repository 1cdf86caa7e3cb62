#!/bin/bash
# Build scripts/tsan_driver with the host runtime under ThreadSanitizer (the sm_100a kernels as
# usual).  Output: build_tsan/tsan_driver.  Run it on the GPU box:
#   TSAN_OPTIONS="halt_on_error=0 second_deadlock_stack=1" build_tsan/tsan_driver
set -e
cd "$(dirname "$0")/.."
C=paper_conf_cgo_panditg14_b200/csrc
O=build_tsan
mkdir -p $O
NVCC=${CUDA_HOME:-/usr/local/cuda}/bin/nvcc
[ -f $O/kernels.o ] || $NVCC -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Xcompiler -fPIC -Iinclude -c $C/kernels.cu -o $O/kernels.o
g++ -std=c++17 -fPIC -O1 -g -fsanitize=thread -march=x86-64-v3 -ffp-contract=off -fno-fast-math -Iinclude -c $C/host_bodies.cpp -o $O/host_bodies.o
g++ -std=c++17 -fPIC -O1 -g -fsanitize=thread -pthread -Iinclude -I${CUDA_HOME:-/usr/local/cuda}/include -c $C/runtime.cpp -o $O/runtime.o
g++ -std=c++17 -O1 -g -fsanitize=thread -pthread -Iinclude -c scripts/tsan_driver.cpp -o $O/tsan_driver.o
$NVCC -gencode arch=compute_100a,code=sm_100a -cudart static -Xcompiler -fsanitize=thread -o $O/tsan_driver \
    $O/tsan_driver.o $O/runtime.o $O/host_bodies.o $O/kernels.o -lpthread -ldl -lrt
echo built $O/tsan_driver
