WLS="M5s-0.3 M5s-0.2 M5s-0.15" ENVS="NONE=0 PTAS_SPEC_LAT_DEPTH=8 PTAS_RING_P2P=1" bash scripts/knob_ab.sh
WLS="M2s M4s" ENVS="NONE=0 PTAS_GRID_DIV=0" bash scripts/knob_ab.sh
