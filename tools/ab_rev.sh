#!/bin/bash
# Build build/ab/NAME.so from the library sources at git revision REV (dev A/B baseline).
#   tools/ab_rev.sh REV NAME ["-DFLAG ..."]
set -e
cd "$(dirname "$0")/.."
rev=$1; name=$2; flags=${3:-}
tmp=$(mktemp -d)
git archive "$rev" paper_conf_hpdc_jaiganeshb18_b200/csrc include | tar -x -C "$tmp"
mkdir -p build/ab
srcs=$(ls "$tmp"/paper_conf_hpdc_jaiganeshb18_b200/csrc/*.cu "$tmp"/paper_conf_hpdc_jaiganeshb18_b200/csrc/*.cpp 2>/dev/null)
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -shared \
  -Xcompiler -fPIC -Xcompiler -fvisibility=hidden -I"$tmp"/include -I"$tmp"/paper_conf_hpdc_jaiganeshb18_b200/csrc \
  $flags $srcs -o build/ab/$name.so
rm -rf "$tmp"
