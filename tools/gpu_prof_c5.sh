# C5 join: ncu --set full with source, plus per-range join times (SJ_DEBUG_VRANGE)
mkdir -p gpurun_out/prof
set -x
timeout 600 ncu --set full --clock-control none --import-source on -k regex:join_kernel -s 2 -c 1 -o gpurun_out/prof/c5_join python tools/step.py c5 2 > gpurun_out/prof/ncu_c5.log 2>&1
tail -3 gpurun_out/prof/ncu_c5.log
python tools/step.py c5 3 2>&1 | tail -1
python - <<'PY' 2>&1 | tail -3
import sys; sys.path.insert(0,'.')
import paper_conf_ipps_galletg19_b200 as sj, workloads, torch
cfg=workloads.get_config('c5'); d=torch.from_numpy(cfg.points()).cuda()
h=sj.Handle(d,cfg.eps,k=8); print('chunks',h.stats()['n_chunks']); h.close()
PY
for r in 0,15000 0,100000 0,300000 300000,2000000 600000,2000000 1000000,2000000; do
  echo "range $r"; SJ_DEBUG_VRANGE=$r python tools/step.py c5 3 2>&1 | tail -1
done
