timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for so in libpsb.so libpsb_mb8.so libpsb_mb10.so libpsb_mb12.so; do
  echo "=== $so"; PSB_LIB_PATH=$PWD/paper_conf_icpp_namkn16_b200/$so timeout 300 python tools/quick_time.py C2 C3 2>&1 | grep -E "psb|bnb|C2|C3"
done
