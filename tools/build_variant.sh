#!/bin/bash
# build an experimental variant of libgraphb.so: tools/build_variant.sh OUT.so -DFLAG ...
out=$1; shift
cd "$(dirname "$0")/../paper_conf_sc_alabanditrb21_b200/csrc"
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared "$@" \
  -o "$out" gb_ingest.cu gb_msbfs.cu gb_tree.cu gb_cycle.cu gb_harary.cu gb_wilson.cu gb_api.cu
