PTAS_LEVEL_TIMES=1 python scripts/level_times.py M2s 3 2>&1 | tail -3
python scripts/level_times.py M2s 3 2>&1 | tail -2
PTAS_DF=0 python scripts/level_times.py M2s 3 2>&1 | tail -2
PTAS_DF=0 PTAS_LEVEL_TIMES=1 python scripts/level_times.py M2s 2 2>&1 | tail -2
