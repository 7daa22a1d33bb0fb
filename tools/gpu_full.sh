set -x
timeout 2400 python -m pytest tests/ -x -q -m gpu 2>&1 | tail -5
timeout 300 python -c "import __graft_entry__ as g; g.smoke()"
timeout 900 python bench.py --steps 20 --warmup 3 2>&1 | tail -1
