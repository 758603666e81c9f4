"""Summarise bench JSON lines (optionally prefixed by a tag): python scripts/show_bench.py file"""
import json, sys
for l in open(sys.argv[1]):
    tag, _, js = l.partition("{")
    try:
        j = json.loads("{" + js)
    except Exception:
        print("unparsed:", l[:160].rstrip()); continue
    r = j.get("roofline", {})
    print(f"{tag.strip():8s} {j['config']['workload']:28s} tile={j['config'].get('tile')!s:4s} {j['value']:8.1f} GCUPS "
          f"{j['ms_per_step']:8.3f} ms  frac={r.get('frac', 0):.3f}  sm={j.get('clocks', {}).get('sm_mhz')}")
