#!/bin/bash
# Build a libgum variant with extra -D flags into build/variants/libgum_<name>.so (tuning aid).
#   tools/build_variant.sh ept16 -DGUM_EPT=16
set -e
name=$1; shift
ROOT=$(cd "$(dirname "$0")/.." && pwd)
mkdir -p "$ROOT/build/variants"
/usr/local/cuda/bin/nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC,-fopenmp,-O3 \
  -I"$ROOT/include" --expt-relaxed-constexpr "$@" -shared -o "$ROOT/build/variants/libgum_$name.so" \
  "$ROOT"/paper_conf_icde_menggltyz23_b200/csrc/*.cu -lgomp
