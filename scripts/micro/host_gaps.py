"""Host scheduling gaps: a tight loop on the clock; reports gaps > 0.5 ms over a few seconds."""
import os, time, sys
dur = float(sys.argv[1]) if len(sys.argv) > 1 else 5.0
t_end = time.perf_counter() + dur
last = time.perf_counter()
gaps = []
while True:
    t = time.perf_counter()
    if t - last > 5e-4:
        gaps.append(t - last)
    last = t
    if t > t_end:
        break
gaps.sort()
print(f"nproc={os.cpu_count()} gaps>0.5ms: {len(gaps)} total {1e3*sum(gaps):.1f} ms in {dur}s; largest {[round(1e3*g,2) for g in gaps[-8:]]}")
