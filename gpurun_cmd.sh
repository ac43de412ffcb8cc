mkdir -p gpurun_out/ncu
for c in C2 C3 C5; do
timeout 900 ncu --set full --import-source on --clock-control none -k regex:psb_kernel --launch-skip 1 -c 1 -f -o gpurun_out/ncu/${c}_psb_v2 python tools/prof_one.py $c psb > gpurun_out/ncu/${c}_psb_v2.log 2>&1
tail -1 gpurun_out/ncu/${c}_psb_v2.log
done
