set -x
O=gpurun_out/r01d; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -3
timeout 600 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err
timeout 900 python bench.py --config C3 > $O/bench_C3.json 2> $O/bench_C3.err
timeout 900 python bench.py --config C4 > $O/bench_C4.json 2> $O/bench_C4.err
timeout 900 python bench.py --config C5 --slab 8 > $O/bench_C5slab8.json 2> $O/bench_C5slab8.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref_C2.json 2> $O/bench_ref_C2.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_c2.csv python bench.py --steps 2 --warmup 3 > $O/launches_run.log 2>&1
for ca in C2:psb C2:bnb C3:psb C3:bnb C4:psb C5:psb; do c=${ca%%:*}; a=${ca##*:}
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"${a}_kernel" --launch-skip 1 -c 1 -f -o $O/prof_${a}_${c} python tools/prof_one.py $c $a > $O/prof_${a}_${c}.log 2>&1
done
ls -la $O
