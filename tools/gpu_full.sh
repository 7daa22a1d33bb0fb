# full GPU check: all gpu tests, smoke, default bench; logs under gpurun_out/
mkdir -p gpurun_out
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
timeout 2400 python -m pytest tests/ -x -q -m gpu --durations=15 > gpurun_out/pytest_gpu.log 2>&1; tail -25 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout 900 python bench.py 2>gpurun_out/bench.err | tee gpurun_out/bench.jsonl | tail -1
