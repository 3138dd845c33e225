# swap in the experimental lib, time, restore
cp paper_conf_sc_tianscd23_b200/libxs.so /tmp/libxs_orig.so
cp exp/libxs.so paper_conf_sc_tianscd23_b200/libxs.so
python tools/quick_time.py --config large --variants sort 2>&1 | tail -1
python tools/quick_time.py --config large-hash --variants sort 2>&1 | tail -1
cp /tmp/libxs_orig.so paper_conf_sc_tianscd23_b200/libxs.so
