timeout 600 python tools/fill_bench.py C2 0 1 3 5 6 8 9 10 11 --reps=2
timeout 600 python tools/fill_bench.py R2000000x536165 0 1 3 5 6 8 9 10 11 --reps=2
