O=gpurun_out/r01al; mkdir -p $O
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1; tail -1 $O/smoke.txt
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -3 > $O/pytest_gpu.txt; cat $O/pytest_gpu.txt
timeout 600 python tools/var_ab.py C5 psb 0 > $O/cf.txt 2>&1
timeout 600 python tools/var_ab.py C2 psb 0 >> $O/cf.txt 2>&1
timeout 900 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err
timeout 1200 python bench.py --config C5 --mode data --slab 8 > $O/bench_C5slab8.json 2> $O/bench_C5slab8.err
timeout 1500 python bench.py --config C5 > $O/bench_C5.json 2> $O/bench_C5.err
cat $O/cf.txt
