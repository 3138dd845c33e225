python exp/repro_explicit.py large 1000000,4000000,8500000,12000000,17000000 dev8 2>&1 | tail -8
python exp/repro_explicit.py large 17000000 dev 2>&1 | tail -3
python exp/repro_explicit.py large 17000000 devns 2>&1 | tail -3
python exp/repro_explicit.py small 17000000 dev8 2>&1 | tail -3
