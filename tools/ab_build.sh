#!/bin/bash
# ab_build.sh NAME "EXTRA NVCC FLAGS" [files...]: rebuild the given .cu files (default tpacf.cu) with
# extra flags, link with the other objects of csrc/build/, write _ab/NAME/libhauberk.so.
set -e
NAME=$1; EXTRA=$2; shift 2; FILES=${@:-tpacf.cu}
ROOT=$(cd "$(dirname "$0")/.." && pwd); C=$ROOT/paper_conf_ipps_yimpski11_b200/csrc
T=/tmp/ab_$NAME; rm -rf $T; mkdir -p $T; cp $C/build/*.o $T/
for f in $FILES; do
  nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -fmad=false -Xcompiler -fPIC \
    -Xcompiler -fvisibility=hidden --expt-relaxed-constexpr $EXTRA -c -o $T/${f%.cu}.o $C/$f
done
mkdir -p $ROOT/_ab/$NAME
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $ROOT/_ab/$NAME/libhauberk.so $T/*.o -Xcompiler -fvisibility=hidden
echo built $ROOT/_ab/$NAME/libhauberk.so
