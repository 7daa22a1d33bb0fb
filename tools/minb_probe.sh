for mb in 2 3 4; do for c in c5 c2k64 c3k64 c4k32; do echo "MINB $mb"; SJ_LIB_PATH=$PWD/paper_conf_ipps_galletg19_b200/libsj_mb$mb.so python tools/step.py $c 2 2>&1 | tail -1; done; done
