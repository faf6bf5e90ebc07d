#!/usr/bin/env python
"""One-line summary of a bench.py JSON line."""
import json
import sys

d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print(f"P={d['config'].get('concurrent_batches_per_gpu')} value={d['value']:.0f} ms/step={d['ms_per_step']:.4f} "
      f"single={d['single_batch']['ms_per_batch']:.4f}ms gather_frac={d['roofline']['frac']:.3f} "
      f"gather_ms={d['roofline']['gather_ms_per_launch']:.4f} e2e={d['e2e']['value']:.0f}")
