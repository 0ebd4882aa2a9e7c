#!/bin/bash
# Build libblastp.so of a commit into ab/<name>.so (for A/B timing): build_commit.sh <name> <commit> [-Dflags]
set -e
name=$1; commit=$2; shift 2
root="$(cd "$(dirname "$0")/.." && pwd)"
tmp=$(mktemp -d)
git -C "$root" archive "$commit" paper_conf_ipps_zhangwlf14_b200/csrc include | tar -x -C "$tmp"
mkdir -p "$root/ab/$name"
for f in "$tmp"/paper_conf_ipps_zhangwlf14_b200/csrc/*.cu; do
  nvcc -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O2 -gencode arch=compute_100a,code=sm_100a -I "$tmp/include" "$@" -c "$f" -o "$root/ab/$name/$(basename $f).o" &
done
wait
nvcc -shared -gencode arch=compute_100a,code=sm_100a -o "$root/ab/$name.so" "$root"/ab/$name/*.o
rm -rf "$tmp"
echo ab/$name.so
