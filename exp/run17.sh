timeout 600 python exp/qt.py 2>&1 || true
