#!/bin/bash
# libbetty variants with other extraction unroll depths into build_var/<name>/libbetty.so
set -e
cd "$(dirname "$0")/../paper_conf_asplos_yangzd023_b200"
for V in ${VARIANTS:-"f2r4:2:4" "f8r4:8:4" "f4r2:4:2" "f4r6:4:6"}; do
  IFS=: read NAME F R <<< "$V"
  mkdir -p build_var/$NAME
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden --expt-relaxed-constexpr -DBETTY_BUILD -DBETTY_FLAT_UNR=$F -DBETTY_RL_UNR=$R -c csrc/extract.cu -o build_var/$NAME/extract.o
  nvcc -gencode arch=compute_100a,code=sm_100a -shared -o build_var/$NAME/libbetty.so build_var/$NAME/extract.o $(ls build/*.o | grep -v '/extract.o') -lcudart
  echo built $NAME
done
