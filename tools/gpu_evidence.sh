# Standard evidence run: gpu tests, smoke, bench lines (all primary configs), ncu launch list of
# the default bench command, one ncu --set full capture of the emitting join launch per primary
# config (summaries kept; the reports are deleted: gpurun_out is capped at 64 MiB).
set -x
OUT=gpurun_out/evidence
mkdir -p $OUT
timeout 2400 python -m pytest tests/ -x -q -m gpu > $OUT/pytest_gpu.log 2>&1; tail -3 $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; tail -1 $OUT/smoke.log
timeout 900 python bench.py --json-out $OUT/bench.jsonl 2>$OUT/bench.err | tail -1
for c in c1 c2k16 c2k64 c2k256 c3k64 c3k256 c4k32 c5e02; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 3 --e2e-steps 1 --no-cpu-baseline --json-out $OUT/bench.jsonl 2>>$OUT/bench.err | tail -1
done
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 --json-out $OUT/bench_ref.jsonl 2>>$OUT/bench.err | tail -1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_bench_c5.csv python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline > $OUT/ncu_launch_run.log 2>&1
for c in c5 c2k64 c3k64 c4k32; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:join_kernel -s 2 -c 1 -o /tmp/prof_${c}_join python tools/step.py $c 2 > $OUT/ncu_${c}.log 2>&1
  python tools/ncu_summary.py /tmp/prof_${c}_join.ncu-rep > $OUT/ncu_${c}_join_summary.txt 2>&1
  ncu -i /tmp/prof_${c}_join.ncu-rep --page raw --csv > $OUT/ncu_${c}_join_raw.csv 2>/dev/null
  rm -f /tmp/prof_${c}_join.ncu-rep
done
ls -la $OUT
