"""Summarise bench JSON lines in a sweep log (label lines followed by JSON lines)."""
import json, sys
for line in open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/s.log"):
    if not line.startswith('{'):
        print(line.strip()); continue
    d = json.loads(line); st = d['stages']
    print(f"  {d['value']:.0f} fps {d['ms_per_step']:.3f} ms conv frac {d['roofline']['frac']:.3f} "
          + " ".join(f"{k}={v['ms_per_step']:.3f}" for k, v in st.items() if isinstance(v, dict)),
          d['counters']['window_hash'])
