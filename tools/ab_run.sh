# A/B join timings in one box: LIBS="a b" CFGS="c5 c3k64" bash tools/ab_run.sh  (exp/libsj_<name>.so)
mkdir -p gpurun_out/r02/ab
for rep in 1 2; do
for c in ${CFGS:-c5}; do for l in ${LIBS}; do
  SJ_LIB_PATH=exp/libsj_$l.so timeout 300 python tools/opt_probe.py $c ${VARS:-default} 2>&1 | sed "s/^/$l /" | tee -a gpurun_out/r02/ab/ab_${TAG:-x}.txt
done; done; done
