# iteration: selected GPU tests (TK), then join/build timings of the primary configs
mkdir -p gpurun_out/r02/iter
timeout ${TT:-1500} python -m pytest ${TPATH:-tests/test_parity_gpu.py} -x -q -m gpu ${TK:+-k "$TK"} > gpurun_out/r02/iter/pytest_${TAG:-it}.log 2>&1; tail -3 gpurun_out/r02/iter/pytest_${TAG:-it}.log
for c in ${CFGS:-c5 c3k64 c2k64 c4k32}; do timeout 120 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline --e2e-steps 0 --batched-steps 0 --json-out gpurun_out/r02/iter/bench_${TAG:-it}.jsonl | python -c "import json,sys; d=json.loads(sys.stdin.readline()); p=d['phases_ms']; print('$c', 'step %.4f build %.4f join %.4f frac %.3f' % (d['ms_per_step'], p['build'], p['join'], d['roofline']['frac']))"; done
