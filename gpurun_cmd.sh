O=gpurun_out/r01am; mkdir -p $O
timeout 900 python bench.py --config C3 > $O/bench_C3.json 2> $O/bench_C3.err
head -c 300 $O/bench_C3.json
