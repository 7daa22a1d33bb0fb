mkdir -p gpurun_out/r02
(nproc; free -g; nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv; python -c "import os; print(len(os.sched_getaffinity(0)))") > gpurun_out/r02/host.txt 2>&1
timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/r02/bench_c5_base.json 2> gpurun_out/r02/bench_c5_base.err
for c in c3k64 c4k32 c5e02; do timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 >> gpurun_out/r02/bench_base.jsonl 2>>gpurun_out/r02/bench_c5_base.err; done
cat gpurun_out/r02/host.txt
