set -x
mkdir -p gpurun_out/ablation
timeout 1200 python tools/ablation.py c2k64 c3k64 c4k32 c5 > gpurun_out/ablation/times.jsonl 2> gpurun_out/ablation/times.err
for c in c2k64 c3k64 c4k32 c5; do
# (the emitting launch, join_kernel<dim, k, kPairs = 1, ...>: the count-only sizing call and the
# SortByWL-only estimator launches are skipped by the name filter)
for v in "gcg input 1 0" "unicomp input 1 0" "lid_unicomp input 1 0" "gcg input 8 0" "gcg workload 1 0" "gcg workload 8 0" "gcg workload 1 1" "gcg workload 8 1" "lid_unicomp workload 8 1"; do
  set -- $v
  timeout 600 ncu --metrics smsp__thread_inst_executed_per_inst_executed.ratio,gpu__time_duration.sum --clock-control none --kernel-name-base demangled -k "regex:join_kernel<[0-9]+, [0-9]+, 1," -c 1 --csv python tools/ablation.py --one $c $1 $2 $3 $4 2>/dev/null | grep -E "thread_inst|duration" | sed "s/^/$c,$1,$2,$3,$4,/" >> gpurun_out/ablation/wee.csv
done; done
