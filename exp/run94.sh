# R=4 (variant 25) vs R=2 (variant 20) staged gather across task densities (N*128/L)
for L in 17000000 12000000 8000000 4000000 2000000; do timeout 300 python exp/cbits.py large 0 5 2 25,20 $L 2>&1; done
for L in 170000000 100000000 60000000; do timeout 600 python exp/cbits.py xl 0 3 2 25,20 $L 2>&1; done
for L in 17000000 4000000; do timeout 300 python exp/cbits.py small 0 5 2 25,20 $L 2>&1; done
