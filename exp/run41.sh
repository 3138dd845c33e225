timeout 600 python tools/quick_time.py --config large --variants sort-v25,sort-v29,sort-v30 --reps 5
timeout 600 python tools/quick_time.py --config large-hash --variants sort-v25,sort-v29,sort-v30 --reps 5
