O=gpurun_out/r02bf; mkdir -p $O
timeout 600 ncu --set full --import-source on --clock-control none -k regex:psb_kernel -s 1 -c 1 -o $O/c5_psb python tools/prof_one.py C5 psb > $O/ncu_c5.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:bnb_kernel -s 1 -c 1 -o $O/c5_bnb python tools/prof_one.py C5 bnb > $O/ncu_c5b.log 2>&1
tail -1 $O/ncu_c5.log $O/ncu_c5b.log
