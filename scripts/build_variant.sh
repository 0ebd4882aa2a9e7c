#!/bin/bash
# Build libblastp.so with extra nvcc flags into ab/<name>.so: build_variant.sh <name> [-Dflags...]
set -e
name=$1; shift
cd "$(dirname "$0")/.."
mkdir -p ab/$name
for f in paper_conf_ipps_zhangwlf14_b200/csrc/*.cu; do
  nvcc -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O2 -gencode arch=compute_100a,code=sm_100a -I include "$@" -c $f -o ab/$name/$(basename $f).o &
done
wait
nvcc -shared -gencode arch=compute_100a,code=sm_100a -o ab/$name.so ab/$name/*.o
echo ab/$name.so
