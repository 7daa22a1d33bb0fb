# quick GPU check: parity (mid-size) + step timings for the primary configs
set -x
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -m gpu -k "not full_size" 2>&1 | tail -5
for c in c5 c2k64 c3k64 c4k32; do timeout 300 python tools/step.py $c 3 2>&1 | tail -2; done
