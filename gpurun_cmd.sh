O=gpurun_out/r02bw; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -x -q > $O/gputests.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1
timeout 600 python bench.py --config C2 > $O/bench_C2.json 2> $O/bench_C2.err
timeout 900 python bench.py --config C5 --mode data --slab 8 --steps 50 > $O/bench_C5slab.json 2> $O/bench_C5slab.err
tail -2 $O/gputests.txt; cat $O/smoke.txt
