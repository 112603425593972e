#!/bin/bash
# Mutation check of the oracle's pins: rebuild oracle.c with one deliberate
# mistake at a time (in a scratch copy under /tmp) and confirm that the CPU pin
# suite (-m "not gpu") fails for every mutation.  Usage: tools/oracle_mutations.sh
set -u
REPO=$(cd "$(dirname "$0")/.." && pwd)
W=/tmp/oracle_mut.$$
mkdir -p $W/oracle
cp -r $REPO/tests $REPO/synth $REPO/pytest.ini $W/
cp $REPO/oracle/__init__.py $W/oracle/
O=$REPO/oracle/oracle.c
declare -a NAME SED
NAME+=("bf16: H_{l+1} not rounded");        SED+=('s/H\[l + 1\].a\[t\] = bf16 ? bf16_round(h) : h;/H[l + 1].a[t] = h;/')
NAME+=("bf16: bias operand not rounded");   SED+=('s|mm_acc(&S, &ones, 0, &bb, 0, bf16);|mm_acc(\&S, \&ones, 0, \&bb, 0, 0);|; s/mat bb = param_mat(params, o.b, 1, fo, bf16);/mat bb = param_mat(params, o.b, 1, fo, 0);/')
NAME+=("project-first rule inverted");      SED+=('s/: (fi > fo);/: (fi <= fo);/')
NAME+=("pool tie: last max wins");          SED+=('s/if (a < 0 || z > best)/if (a < 0 || z >= best)/')
NAME+=("REG: diagonal kept");               SED+=('s/if (j == i) continue;/if (0) continue;/')
NAME+=("mean: 1/D dropped in backward");    SED+=('s|AT(dA, v, f) / (double)deg;|AT(dA, v, f);|')
NAME+=("loss scale dropped from dS");       SED+=('s/AT(dS, v, c) = loss_scale \* (/AT(dS, v, c) = (/')
NAME+=("ReLU mask dropped in backward");    SED+=('s/if (!(X.a\[t\] > 0.0)) dX.a\[t\] = 0.0;/;/')
fail=0
for i in "${!NAME[@]}"; do
  cp $O $W/oracle/oracle.c
  sed -i "${SED[$i]}" $W/oracle/oracle.c
  if cmp -s $O $W/oracle/oracle.c; then echo "SKIP (pattern not found): ${NAME[$i]}"; fail=1; continue; fi
  rm -f $W/oracle/liboracle.so
  r=$(cd $W && python -m pytest -q -x -p no:cacheprovider tests/test_oracle_*.py -m "not gpu" 2>&1 | tail -1)
  case "$r" in *failed*) echo "caught   : ${NAME[$i]} -- $r";; *) echo "SURVIVED : ${NAME[$i]} -- $r"; fail=1;; esac
done
rm -rf $W
exit $fail
