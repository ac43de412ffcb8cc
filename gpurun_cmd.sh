set -x
O=gpurun_out/r01n; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -3 > $O/pytest_gpu.txt; cat $O/pytest_gpu.txt
for c in C2 C3 C4 C5 C5W; do timeout 900 python tools/var_ab.py $c psb 0 128 > $O/kth_$c.txt 2>&1; done
for c in C2 C4; do timeout 900 python tools/var_ab.py $c bnb 0 128 > $O/kth_${c}_bnb.txt 2>&1; done
cat $O/kth_*
