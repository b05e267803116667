#!/bin/bash
# Build variant libraries with extra nvcc flags into build/ab/<name>.so (dev A/B tests).
#   tools/ab.sh NAME "-DFLAG=..." [NAME2 "-D..."]...
set -e
cd "$(dirname "$0")/.."
mkdir -p build/ab
while [ $# -ge 2 ]; do
  name=$1; flags=$2; shift 2
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -shared \
    -Xcompiler -fPIC -Xcompiler -fvisibility=hidden -Iinclude -Ipaper_conf_hpdc_jaiganeshb18_b200/csrc \
    $flags paper_conf_hpdc_jaiganeshb18_b200/csrc/ecl_cc.cu paper_conf_hpdc_jaiganeshb18_b200/csrc/ecl_cc_csr.cu paper_conf_hpdc_jaiganeshb18_b200/csrc/ecl_cc_io.cpp -o build/ab/$name.so &
done
wait
