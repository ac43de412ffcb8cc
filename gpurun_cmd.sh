O=gpurun_out/r02bq; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -x -q > $O/gputests.txt 2>&1
for r in 1 2; do for c in C2 C5 C3; do
  PSB_LIB_PATH=$PWD/paper_conf_icpp_namkn16_b200/libpsb_base.so timeout 300 python tools/var_ab.py $c psb 0 > $O/ab_base_${c}_$r.txt 2>&1
  timeout 300 python tools/var_ab.py $c psb 0 > $O/ab_new_${c}_$r.txt 2>&1
done; done
tail -2 $O/gputests.txt; for f in $O/ab_*; do echo "$f $(tail -1 $f | cut -c1-40)"; done
