"""Print bench JSON lines compactly: workload dtype variant GFLOPS ms per-kernel ms/fraction."""
import json
import sys

for path in sys.argv[1:]:
    for l in open(path):
        if not l.startswith('{'):
            print('   ', l.strip())
            continue
        d = json.loads(l)
        c, r = d['config'], d.get('roofline') or {}
        peak = r.get('peak') or 6461.0
        ks = ' | '.join(f"{k[5:]} {v['avg_ms']:.4f}ms {(v['alg_gbs'] or 0) / peak:.3f}" for k, v in (r.get('kernels') or {}).items())
        print(c.get('workload'), d['dtype'], c.get('variant'), round(d['value'], 1), 'ms', round(d['ms_per_step'], 4),
              'eff', round(d.get('effective_frac_of_peak') or 0, 3), ks)
