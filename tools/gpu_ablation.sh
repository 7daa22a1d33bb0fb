set -x
mkdir -p gpurun_out/ablation
[ -n "$NO_TIMES" ] || timeout 1200 python tools/ablation.py c2k64 c3k64 c4k32 c5 > gpurun_out/ablation/times.jsonl 2> gpurun_out/ablation/times.err
for c in c2k64 c3k64 c4k32 c5; do
for v in "gcg input 1 0" "unicomp input 1 0" "lid_unicomp input 1 0" "gcg input 8 0" "gcg workload 1 0" "gcg workload 8 0" "gcg workload 1 1" "gcg workload 8 1" "lid_unicomp workload 8 1"; do
  set -- $v
  skip=$([ "$4" = "0" ] && echo 2 || echo 1)  # launches before the emitting join: the count-only
  # sizing call, plus the estimator when the sample is strided (SortByWL only, queue 0)
  timeout 600 ncu --metrics smsp__thread_inst_executed_per_inst_executed.ratio,gpu__time_duration.sum --clock-control none -k regex:join_kernel -s $skip -c 1 --csv python tools/ablation.py --one $c $1 $2 $3 $4 2>/dev/null | grep -E "thread_inst|duration" | sed "s/^/$c,$1,$2,$3,$4,/" >> gpurun_out/ablation/wee.csv
done; done
