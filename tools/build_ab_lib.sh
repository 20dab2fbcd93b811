#!/bin/bash
# Build a libsvp variant for an A/B run: every object of the current build except the given
# kernel source, which is taken from a git revision.   tools/build_ab_lib.sh <rev> <kernels/x.cu> <out.so>
set -e
rev=$1; src=$2; out=$3
root=$(cd "$(dirname "$0")/.." && pwd)
python -m paper_conf_dac_jungc15_b200._build > /dev/null
tmp=$(mktemp -d)
git -C "$root" show "$rev:paper_conf_dac_jungc15_b200/csrc/$src" > "$tmp/ab.cu"
sed -i "s#\"../launch.h\"#\"$root/paper_conf_dac_jungc15_b200/csrc/launch.h\"#; s#\"common.cuh\"#\"$root/paper_conf_dac_jungc15_b200/csrc/kernels/common.cuh\"#" "$tmp/ab.cu"
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -I"$root/include" -c "$tmp/ab.cu" -o "$tmp/ab.o"
base=$(basename "$src" .cu)
objs=$(ls "$root"/build/svp/*.o | grep -v "kernels_${base}.cu.o")
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o "$out" $objs "$tmp/ab.o" -cudart static -lpthread -ldl -lrt
rm -rf "$tmp"
echo "$out"
