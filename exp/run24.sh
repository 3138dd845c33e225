timeout 600 python exp/qt3.py large 0 26 27 24 19 2>&1
