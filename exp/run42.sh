timeout 600 python tools/quick_time.py --config large --variants sort-v25 --reps 10
timeout 600 python tools/quick_time.py --config small --variants sort-v25 --reps 10
