# blocked-output join time per block size (SJ_OUT_BLK) for C5 and C2K64
for b in 1024 2048 4096 8192; do echo "blk $b"; SJ_OUT_BLK=$b python tools/blk_probe.py ${1:-c5} 5; done
