#!/usr/bin/env python
"""One-line summary of a bench.py JSON line."""
import json
import sys

d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
ns = d.get("north_star_workload") or {}
par = d.get("parity") or {}
print(f"N={d['n_gpus']} P={d['config'].get('concurrent_batches_per_gpu')} value={d['value']:.0f} "
      f"ms/step={d['ms_per_step']:.4f} single={d['single_batch']['ms_per_batch']:.4f}ms "
      f"gather_frac={d['roofline']['frac']:.3f} ({d['roofline']['bound']}) "
      f"whole_step={d.get('whole_step_roofline', {}).get('frac', 0):.3f} e2e={d['e2e']['value']:.0f} "
      f"parity={par.get('ok')} clocks={(d.get('clocks') or {}).get('sm_mhz')} "
      + (f"papers={ns['value']:.0f} papers_frac={ns['roofline']['frac']:.3f} papers_parity={ns['parity']['ok']}"
         if ns else ""))
