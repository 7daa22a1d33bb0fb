# Round-2 evidence run: GPU tests, smoke, bench lines for every config (default first), the
# reference arm, the ncu launch list of the default bench command, and per config one
# `ncu --set full` capture of the emitting join launch + the build kernels' DRAM bytes.
OUT=gpurun_out/r02/ev${EVTAG:-}
mkdir -p $OUT
if [ -z "$NOTESTS" ]; then
timeout 2400 python -m pytest tests/ -x -q -m gpu > $OUT/pytest_gpu.log 2>&1; tail -3 $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; tail -1 $OUT/smoke.log
fi
for c in ${CFGS:-c5 c2k64 c3k64 c4k32 c5e02 c1 c2k16 c2k256 c3k256}; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:join_kernel -s 1 -c 1 -o /tmp/prof_${c}_join python tools/step.py $c 2 > $OUT/ncu_${c}.log 2>&1
  python tools/ncu_summary.py /tmp/prof_${c}_join.ncu-rep > $OUT/ncu_${c}_join_summary.txt 2>&1
  ncu -i /tmp/prof_${c}_join.ncu-rep --page raw --csv > $OUT/ncu_${c}_join_raw.csv 2>/dev/null
  rm -f /tmp/prof_${c}_join.ncu-rep
  timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv --log-file $OUT/ncu_${c}_build_metrics_all.csv python tools/step.py $c 1 > /dev/null 2>&1
  python tools/last_step_kernels.py $OUT/ncu_${c}_build_metrics_all.csv > $OUT/ncu_${c}_build_metrics.csv 2>/dev/null
done
python tools/r02_facts.py $OUT r02/ev${EVTAG:-} > $OUT/facts.json 2>&1; cp profiles/ncu_facts.json $OUT/ncu_facts.json
timeout 900 python bench.py --json-out $OUT/bench.jsonl 2>$OUT/bench.err | tail -1
for c in ${BCFGS:-c2k64 c3k64 c4k32 c5e02 c1 c2k16 c2k256 c3k256}; do
  timeout 600 python bench.py --config $c --steps 30 --warmup 3 --e2e-steps 1 --batched-steps 2 --no-cpu-baseline --json-out $OUT/bench.jsonl 2>>$OUT/bench.err | tail -c 300
done
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 --json-out $OUT/bench_ref.jsonl 2>>$OUT/bench.err | tail -c 300
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_bench_c5.csv python bench.py --steps 2 --warmup 1 --e2e-steps 0 --batched-steps 0 --no-cpu-baseline > $OUT/ncu_launch_run.log 2>&1
python tools/launch_summary.py $OUT/launches_bench_c5.csv > $OUT/launches_bench_c5_summary.txt 2>&1
ls $OUT | head -80
