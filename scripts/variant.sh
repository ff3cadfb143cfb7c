#!/bin/bash
# Build a variant of libspgemm.so with one source recompiled under extra defines (A/B runs via
# SPGEMM_LIB=variants/NAME.so).  The in-tree build must be current (python -m ...build).
#   bash scripts/variant.sh NAME SOURCE.cu [-DX=Y ...]
set -e
NAME=$1; SRC=$2; shift 2
B=paper_conf_icpp_nagasakanm17_b200/_build
mkdir -p variants/$NAME.o.d
nvcc -O3 -std=c++17 -lineinfo -gencode arch=compute_100a,code=sm_100a -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
  --expt-relaxed-constexpr -Iinclude -Ipaper_conf_icpp_nagasakanm17_b200/csrc -Xptxas -v "$@" -c "$SRC" \
  -o variants/$NAME.o.d/var.o 2> variants/$NAME.ptxas.log
STEM=$(basename "$SRC" .cu)
OBJS=$(ls $B/*.o | grep -v "/$STEM.o$")
nvcc -shared -gencode arch=compute_100a,code=sm_100a -o variants/$NAME.so $OBJS variants/$NAME.o.d/var.o
echo variants/$NAME.so
