#!/bin/bash
# bench-only A/B of library variants (each run twice, interleaved)
for rep in 1 2; do
for lib in "$@"; do
  printf "%-28s " "$(basename $lib)"
  PHMM_LIB=$lib python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']
print('step GCUPS %.0f ms/step %.2f'%(d['value'], d['ms_per_step']), 'wavefront %.2f ms'%r['wavefront_ms'], 'kernel GCUPS %.0f frac %.3f'%(r['achieved'], r['frac']), 'clk', d['clocks'].get('sm_mhz'))"
done; done
