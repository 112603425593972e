#!/bin/bash
# build_variant.sh NAME SRC DEF[,DEF...]: libbetty.so with one source file recompiled under extra
# -D definitions, into build_var/NAME/ (A/B runs select it with BETTY_LIB_PATH; tools/ab.sh)
set -e
cd "$(dirname "$0")/../paper_conf_asplos_yangzd023_b200"
NAME=$1; SRC=$2; DEFS=$3
XDEF=""; [ -n "$DEFS" ] && XDEF="-D${DEFS//,/ -D}"
mkdir -p build_var/$NAME
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden --expt-relaxed-constexpr -Xptxas -v -DBETTY_BUILD $XDEF -c csrc/$SRC.cu -o build_var/$NAME/$SRC.o 2> build_var/$NAME/ptxas.log
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o build_var/$NAME/libbetty.so build_var/$NAME/$SRC.o $(ls build/*.o | grep -v "/$SRC.o") -lcudart
echo built $NAME
