import json, sys
for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "ERR", e); continue
    c = d["config"]
    print(f"{c['workload']:<22} {d['value']:9.1f} GFLOPS  {d['ms_per_step']:9.3f} ms  steps {c['step_ms']}  alloc {c.get('alloc_sync_ms')}  roof {d['roofline']['frac']:.3f} ({d['roofline']['kernel']})")
