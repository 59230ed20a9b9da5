#!/bin/bash
# ASan + UBSan build of the host code (netlist, compiler, collapse, tile planner) and of the
# C oracle, then the CPU test suite against them.  Runs on the CPU box.
set -e
cd "$(dirname "$0")/.."
OUT=build_asan
mkdir -p $OUT
SAN="-fsanitize=address,undefined -fno-omit-frame-pointer -fno-sanitize-recover=undefined -g -O1"
ARCH="-gencode arch=compute_100a,code=sm_100a"
objs=""
BID=$(python -c "import paper_conf_ipps_gavierrprs23_b200._build as b; print(b.build_id())")
for f in paper_conf_ipps_gavierrprs23_b200/csrc/*.cpp; do
  o=$OUT/$(basename $f).o
  g++ -std=c++17 -Iinclude -I/usr/local/cuda/include -fPIC $SAN -DGS_BUILD_ID=\"$BID\" -c $f -o $o
  objs="$objs $o"
done
for f in paper_conf_ipps_gavierrprs23_b200/csrc/*.cu; do
  o=$OUT/$(basename $f).o
  nvcc $ARCH -O3 -std=c++17 -Iinclude -Xcompiler -fPIC -c $f -o $o
  objs="$objs $o"
done
nvcc $ARCH -shared -o $OUT/libgsim.so $objs -cudart static -lasan -lubsan
gcc -std=c11 -fopenmp -fPIC -shared $SAN -o $OUT/liboracle.so oracle/oracle.c
# swap the instrumented libraries in, run the CPU suite, restore
cp paper_conf_ipps_gavierrprs23_b200/libgsim.so $OUT/libgsim.so.orig
cp oracle/liboracle.so $OUT/liboracle.so.orig
cp $OUT/libgsim.so paper_conf_ipps_gavierrprs23_b200/libgsim.so
cp $OUT/liboracle.so oracle/liboracle.so
touch paper_conf_ipps_gavierrprs23_b200/libgsim.so oracle/liboracle.so
set +e
LD_PRELOAD="$(gcc -print-file-name=libasan.so) $(gcc -print-file-name=libubsan.so)" \
  ASAN_OPTIONS=detect_leaks=0,halt_on_error=1 UBSAN_OPTIONS=halt_on_error=1,print_stacktrace=1 \
  python -m pytest tests -q -m "not gpu" -x -p no:cacheprovider "$@"
rc=$?
cp $OUT/libgsim.so.orig paper_conf_ipps_gavierrprs23_b200/libgsim.so
cp $OUT/liboracle.so.orig oracle/liboracle.so
touch paper_conf_ipps_gavierrprs23_b200/libgsim.so oracle/liboracle.so
exit $rc
