O=gpurun_out/r02dp; mkdir -p $O
for r in 1 2; do for c in C3 C4; do
  timeout 300 python tools/var_ab.py $c psb 0 > $O/ab_base_${c}_$r.txt 2>&1
  PSB_LIB_PATH=$PWD/paper_conf_icpp_namkn16_b200/libpsb_pp.so timeout 300 python tools/var_ab.py $c psb 0 > $O/ab_pp_${c}_$r.txt 2>&1
done; done
for f in $O/ab_*; do echo "$f $(tail -1 $f | cut -c1-40)"; done
