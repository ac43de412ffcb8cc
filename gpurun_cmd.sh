O=gpurun_out/r02dk; mkdir -p $O
for s in 2 4 8; do timeout 900 python bench.py --config C3 --mode data --slab $s --steps 50 --no-cpu-baseline --no-extras > $O/bench_C3_slab$s.json 2> $O/bench_C3_slab$s.err; done
for f in $O/*.json; do echo $f; head -c 250 $f; echo; done
