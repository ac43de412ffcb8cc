for c in C2 C3 C5; do
for a in psb bnb; do
PSB_LIB_PATH=$PWD/ab/libpsb_prev.so timeout 300 python tools/var_ab.py $c $a 0 2>&1 | grep -v Warn | sed 's/^/PREV /'
timeout 300 python tools/var_ab.py $c $a 0 2>&1 | grep -v Warn
done; done
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
