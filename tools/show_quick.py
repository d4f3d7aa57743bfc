import json, sys
for line in open(sys.argv[1] if len(sys.argv) > 1 else 'gpurun_out/quick.jsonl'):
    try: d = json.loads(line)
    except Exception: continue
    c = d['config']
    print(f"{c['workload']:16s} {c['mode']:12s} {'sorted' if c['sorted'] else 'unsorted':8s} kern={d['traverse_ms']:9.3f} ms step={d['ms_per_step']:9.3f} pts/s={d['value']:.4g} visits/pt={d['visits_per_point']:.0f} lock={d['lockstep_warp_fraction']:.2f}")
