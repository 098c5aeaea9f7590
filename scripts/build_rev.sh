# build libgem.so of a git revision into exp_libs/libgem_<name>.so (A/B timing on one box)
# usage: bash scripts/build_rev.sh <rev> <name>
set -e
R=$(cd "$(dirname "$0")/.." && pwd)
T=$(mktemp -d)
for f in gem_runtime.cu gem_lanes.cuh gem_isa.h; do git -C "$R" show "$1:paper_conf_dac_guozwlr25_b200/csrc/$f" > "$T/$f"; done
git -C "$R" show "$1:include/gem.h" > "$T/gem.h"
mkdir -p "$R/exp_libs"
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -shared -Xcompiler -fPIC -I "$T" -o "$R/exp_libs/libgem_$2.so" "$T/gem_runtime.cu"
rm -rf "$T"
