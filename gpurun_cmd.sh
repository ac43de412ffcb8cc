timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
QT_FLAGS=--build timeout 900 python tools/quick_time.py C2 C3 C4 2>&1
