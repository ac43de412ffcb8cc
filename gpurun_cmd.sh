set -x
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
timeout 600 python bench.py 2>&1 | tail -1 > gpurun_out/bench_c2.json; cat gpurun_out/bench_c2.json
timeout 400 python tools/quick_time.py C1 C2 C3 2>&1 | tail -30
