#!/bin/bash
# A/B experiments: build libsj.so from git revision REV (or the working tree: "wt") into
# exp/libsj_NAME.so; run with SJ_LIB_PATH=exp/libsj_NAME.so.   usage: tools/ab_build.sh NAME [REV] [EXTRA nvcc flags]
set -e
NAME=$1; REV=${2:-wt}; EXTRA=${3:-}
ROOT=$(cd "$(dirname "$0")/.." && pwd)
T=/tmp/ab_$NAME; rm -rf $T; mkdir -p $T/paper_conf_ipps_galletg19_b200 $T/include
if [ "$REV" = "wt" ]; then
  cp -r $ROOT/paper_conf_ipps_galletg19_b200/csrc $T/paper_conf_ipps_galletg19_b200/; cp $ROOT/include/sj.h $T/include/
else
  git -C $ROOT archive $REV paper_conf_ipps_galletg19_b200/csrc include | tar -x -C $T
fi
rm -rf $T/paper_conf_ipps_galletg19_b200/csrc/build
mkdir -p $ROOT/exp
make -C $T/paper_conf_ipps_galletg19_b200/csrc -j16 OUT=$ROOT/exp/libsj_$NAME.so EXTRA="$EXTRA" > $T/build.log 2>&1 || (tail -20 $T/build.log; exit 1)
echo built $ROOT/exp/libsj_$NAME.so
