#!/bin/bash
# Build an A/B variant of libgsnp.so: tools/build_variant.sh NAME -DFLAG=V ...
# -> paper_conf_icpp_luzlwfl11_b200/libgsnp_NAME.so (load with GSNP_LIB=...)
NAME=$1; shift
D=paper_conf_icpp_luzlwfl11_b200
nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo --fmad=false \
    -Xcompiler -fPIC,-ffp-contract=off -shared -Iinclude "$@" -o $D/libgsnp_$NAME.so \
    $D/csrc/gsnp.cu $D/csrc/gsnp_deep.cu
