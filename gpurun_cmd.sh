timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
mkdir -p gpurun_out/r01c
timeout 600 python bench.py > gpurun_out/r01c/bench_C2.json 2> gpurun_out/r01c/bench_C2.err; tail -c 3000 gpurun_out/r01c/bench_C2.json
timeout 900 python bench.py --config C3 --steps 30 > gpurun_out/r01c/bench_C3.json 2> gpurun_out/r01c/bench_C3.err; tail -c 3000 gpurun_out/r01c/bench_C3.json
timeout 900 python bench.py --config C4 --steps 20 --no-cpu-baseline > gpurun_out/r01c/bench_C4.json 2> gpurun_out/r01c/bench_C4.err; tail -c 3000 gpurun_out/r01c/bench_C4.json
timeout 1500 python bench.py --config C5 --mode data --slab 8 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/r01c/bench_C5slab8.json 2> gpurun_out/r01c/bench_C5slab8.err; tail -c 3000 gpurun_out/r01c/bench_C5slab8.json; tail -5 gpurun_out/r01c/bench_C5slab8.err
