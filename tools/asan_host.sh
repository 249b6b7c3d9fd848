#!/bin/bash
# AddressSanitizer + UBSan build of libkfuse's host code (planner, code
# generator, C-ABI; the CUDA runtime parts are built by nvcc with ASan on the
# host side) and a drive over the planners and the code generator (no GPU).
set -e
cd "$(dirname "$0")/.."
OUT=/tmp/kf_asan; mkdir -p $OUT
SRC=paper_conf_cgo_qiaorht19_b200/csrc
for f in capi.cpp graph.cpp planner.cpp codegen.cpp; do
  g++ -std=c++17 -O1 -g -fsanitize=address,undefined -fno-omit-frame-pointer -fPIC -Iinclude -I$SRC -I/usr/local/cuda/include -c $SRC/$f -o $OUT/$f.o
done
for f in runtime.cu peer.cu; do
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -std=c++17 -O1 -g -Xcompiler -fPIC,-fsanitize=address,-fno-omit-frame-pointer -Iinclude -I$SRC -c $SRC/$f -o $OUT/$f.o
done
g++ -shared -fsanitize=address,undefined -o $OUT/libkfuse.so $OUT/*.o -L/usr/local/cuda/lib64 -lnvrtc -lcudart_static -ldl -lrt -lpthread -Wl,-rpath=/usr/local/cuda/lib64
ASAN_OPTIONS=detect_leaks=0,halt_on_error=1 UBSAN_OPTIONS=halt_on_error=1,print_stacktrace=1 \
  LD_PRELOAD=$(gcc -print-file-name=libasan.so):$(gcc -print-file-name=libubsan.so) \
  KF_ASAN_LIB=$OUT/libkfuse.so python tools/asan_drive.py
