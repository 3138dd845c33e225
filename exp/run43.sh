python exp/h2d_bw.py
timeout 600 python tools/e2e_sweep.py 17000000 4250000 2125000 1062500
