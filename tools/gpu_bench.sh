# full-size parity + first bench + launch list + ncu capture of the join kernel
set -x
timeout 1200 python -m pytest tests/test_parity_gpu.py -x -q -m gpu -k "full_size" 2>&1 | tail -15
timeout 600 python bench.py --steps 20 --warmup 3 --json-out gpurun_out/bench_c5.jsonl 2>&1 | tail -3
for c in c2k64 c3k64 c4k32; do timeout 600 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 1 --no-cpu-baseline --json-out gpurun_out/bench_$c.jsonl 2>&1 | tail -1; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c5.csv python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu_launch_run.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:join_kernel -s 1 -c 1 -o gpurun_out/prof_c5 python bench.py --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu_full_run.log 2>&1
ls -la gpurun_out
