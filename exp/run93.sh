# staged-gather configuration sweep at XL size
timeout 1200 python exp/cbits.py xl 0 3 2 0,17,18,19,20,21,22,23,24,26,27,28 2>&1
