O=gpurun_out/r02ba; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $O/gputests.txt 2>&1
timeout 600 python bench.py > $O/bench_C3.json 2> $O/bench_C3.err
tail -3 $O/gputests.txt; cat $O/smoke.txt; head -c 400 $O/bench_C3.json
