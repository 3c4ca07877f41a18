WLS="M2s M4s M4x M3g" ENVS="NONE=0 PTAS_LIB=variants/minb4/libptas_b200.so" bash scripts/knob_ab.sh
