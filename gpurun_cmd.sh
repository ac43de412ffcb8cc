for rep in 1 2; do
for so in libpsb_base.so libpsb.so libpsb_skip.so; do
  echo "=== $so"; PSB_LIB_PATH=$PWD/paper_conf_icpp_namkn16_b200/$so timeout 300 python tools/quick_time.py C2 C3 2>&1 | grep -E "psb  "
done; done
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
