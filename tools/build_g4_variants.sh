#!/bin/bash
# build libbetty variants with other gather4 pipeline shapes into build_var/<name>/libbetty.so
set -e
cd "$(dirname "$0")/../paper_conf_asplos_yangzd023_b200"
for V in ${VARIANTS:-"m8:8:4:4:8:64" "m32:8:4:4:32:64" "cl32:8:4:4:16:32" "cl128:8:4:4:16:128"}; do
  IFS=: read NAME S P C MR CL X1 <<< "$V"
  XDEF=""; [ -n "$X1" ] && XDEF="-D${X1//,/ -D}"
  mkdir -p build_var/$NAME
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden --expt-relaxed-constexpr -DBETTY_BUILD -DBETTY_G4_STAGES=$S -DBETTY_G4_PROD=$P -DBETTY_G4_CPP=$C -DBETTY_G4_MAXR=$MR -DBETTY_G4_CLAIM=$CL $XDEF -c csrc/agg.cu -o build_var/$NAME/agg.o
  nvcc -gencode arch=compute_100a,code=sm_100a -shared -o build_var/$NAME/libbetty.so build_var/$NAME/agg.o $(ls build/*.o | grep -v '/agg.o') -lcudart
  echo built $NAME
done
