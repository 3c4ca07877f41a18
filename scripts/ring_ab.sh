# ring kernel A/B: parity, per-DP times (barrier vs point-to-point, extra slots), solve benches
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ring.py -m gpu -q -x > gpurun_out/ra_test.log 2>&1; echo ring tests rc=$?; tail -3 gpurun_out/ra_test.log
for W in M5s-0.3 M5s-0.2; do
  for cfg in ${CFGS:-"0 0" "1 0" "1 1" "1 2" "1 4" "1 8"}; do
    set -- ${cfg/_/ }
    echo "== $W P2P=$1 EXTRA=$2"; PTAS_RING_P2P=$1 PTAS_RING_EXTRA=$2 python scripts/ring_prof.py $W 6 2>&1 | tail -3
  done
  PTAS_LIB=variants/ringprof/libptas_b200.so python scripts/ring_prof.py $W 2 2>&1 | grep -v "^  L=" | tail -4
  PTAS_RING_P2P=0 PTAS_LIB=variants/ringprof/libptas_b200.so python scripts/ring_prof.py $W 2 2>&1 | grep -v "^  L=" | tail -4
done
for W in M5s-0.3 M5s-0.2; do
  for p2p in 0 1; do
    PTAS_RING_P2P=$p2p timeout 300 python bench.py --workload $W --no-cpu-baseline --steps 10 --warmup 3 > gpurun_out/ra_b_${W}_$p2p.log 2>&1
    tail -1 gpurun_out/ra_b_${W}_$p2p.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$W p2p=$p2p solve %.3f ms fill %.3f ms frac %.3f parity %s' % (d['ms_per_step'], r['fill_ms_per_step'], r['frac'], d['parity']['solve']['match']))"
  done
done
