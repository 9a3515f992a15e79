#!/bin/bash
# A/B of library variants on C2 and C3 (each lib twice, interleaved): step GCUPS, FP32 kernel
# GCUPS and roofline fraction, rescue ms
WL=${WL:-C2 C3}
for rep in 1 2; do
for wl in $WL; do
for lib in "$@"; do
  printf "%-6s %-28s " $wl "$(basename $lib)"
  PHMM_LIB=$lib python bench.py --workload $wl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-extra 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; q=d['rescue']
print('step %.0f ms %.2f'%(d['value'], d['ms_per_step']), 'wf %.2f ms kernel %.0f frac %.3f'%(r['wavefront_ms'], r['achieved'], r['frac']), 'rescue %.2f ms frac %.3f'%(q['ms'], q['frac'] or 0), 'clk', d['clocks'].get('sm_mhz'))"
done; done; done
