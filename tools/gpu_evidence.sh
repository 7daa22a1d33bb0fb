# Standard evidence run: bench lines (all primary configs), ncu launch list of the default
# bench command, one ncu --set full capture of the emitting join launch per primary config.
set -x
OUT=gpurun_out/evidence
mkdir -p $OUT
timeout 900 python bench.py --steps 20 --warmup 3 --json-out $OUT/bench.jsonl 2>&1 | tail -1
for c in c1 c2k16 c2k64 c2k256 c3k64 c3k256 c4k32 c5e02; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 1 --no-cpu-baseline --json-out $OUT/bench.jsonl 2>&1 | tail -1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_bench_c5.csv python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline > $OUT/ncu_launch_run.log 2>&1
for c in c5 c2k64 c3k64 c4k32; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:join_kernel -s 2 -c 1 -o $OUT/prof_${c}_join python tools/step.py $c 2 > $OUT/ncu_${c}.log 2>&1
done
ls -la $OUT
