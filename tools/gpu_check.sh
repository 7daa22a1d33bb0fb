set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
nproc
python -c "
import sys; sys.path.insert(0,'.')
import paper_conf_ipps_galletg19_b200 as sj, torch
torch.cuda.init()
print('fp64', sj.sj_measure_fp64())
print('fp64', sj.sj_measure_fp64())
print('atomics', sj.sj_measure_atomics())
print('atomics', sj.sj_measure_atomics())
"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()"
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -m gpu -k "not full_size" 2>&1 | tail -30
