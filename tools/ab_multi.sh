#!/bin/bash
# bench-only A/B of library variants on several workloads (each run twice, interleaved)
# usage: WORKLOADS="C2 C5" tools/ab_multi.sh lib1.so lib2.so ...
for w in ${WORKLOADS:-C2}; do
for rep in 1 2; do
for lib in "$@"; do
  printf "%-4s %-24s " "$w" "$(basename $lib)"
  PHMM_LIB=$lib python bench.py --workload $w --steps 5 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; q=d.get('rescue') or {}
print('step GCUPS %.0f ms/step %.2f'%(d['value'], d['ms_per_step']), 'wf %.2f ms'%r['wavefront_ms'], 'kernel %.0f frac %.3f'%(r['achieved'], r['frac']), 'rescue %.2f ms'%q.get('ms', 0), 'clk', d['clocks'].get('sm_mhz'))"
done; done; done
