# k_part_fine window size sweep (two blocks per SM below ~11.5k energies)
export FINE_CAPS=0,11264,10240,8192
timeout 600 python exp/cbits.py large 0 10 2>&1
timeout 600 python exp/cbits.py small 0 10 2>&1
timeout 900 python exp/cbits.py xl 0 3 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "cbits or sorted or explicit" 2>&1 | tail -1
