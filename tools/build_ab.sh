#!/bin/bash
# Build A/B variants of libzh: tools/build_ab.sh name "-DFLAG=V ..." -> ab/libzh_<name>.so
set -e
mkdir -p ab
SRCS=$(python -c "
from paper_conf_ipps_zhangw14_b200 import _build as b; import os; print(' '.join(os.path.join(b.CSRC,s) for s in b.SOURCES))")
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared -Xptxas -O3 $2 $SRCS -o ab/libzh_$1.so
