#!/bin/bash
# build libbetty variants with other gather4 pipeline shapes into build_var/<name>/libbetty.so
set -e
cd "$(dirname "$0")/../paper_conf_asplos_yangzd023_b200"
for V in "s8p4c5:8:4:5" "s8p4c6:8:4:6" "s8p2c6:8:2:6" "s8p4c7:8:4:7"; do
  IFS=: read NAME S P C <<< "$V"
  mkdir -p build_var/$NAME
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden --expt-relaxed-constexpr -DBETTY_BUILD -DBETTY_G4_STAGES=$S -DBETTY_G4_PROD=$P -DBETTY_G4_CPP=$C -c csrc/agg.cu -o build_var/$NAME/agg.o
  nvcc -gencode arch=compute_100a,code=sm_100a -shared -o build_var/$NAME/libbetty.so build_var/$NAME/agg.o $(ls build/*.o | grep -v '/agg.o') -lcudart
  echo built $NAME
done
