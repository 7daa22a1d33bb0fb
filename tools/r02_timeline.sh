mkdir -p gpurun_out/r02/tl
for c in ${CFGS:-c5 c3k64 c1}; do timeout 300 python tools/timeline.py $c 3 > gpurun_out/r02/tl/tl_$c.txt 2>&1; tail -4 gpurun_out/r02/tl/tl_$c.txt; done
timeout 300 python bench.py --steps 30 --warmup 3 --no-cpu-baseline --e2e-steps 0 --batched-steps 0 | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print(d['ms_per_step'], d['phases_ms'])"
