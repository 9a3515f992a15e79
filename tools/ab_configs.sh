#!/bin/bash
# GPU tests, then the bench on C2..C5 for each library given (default: the in-tree one)
python -m pytest tests -m gpu -q -x 2>&1 | tail -2
libs="$@"; [ -z "$libs" ] && libs=paper_conf_ipps_wangxc17_b200/libphmm.so
for lib in $libs; do
 for w in C2 C3 C4 C5; do
  PHMM_LIB=$lib python bench.py --workload $w --steps 4 --warmup 2 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; q=d['rescue']
print('$(basename $lib) $w step GCUPS %.0f ms/step %.2f'%(d['value'], d['ms_per_step']), 'wf %.2f ms %.0f GCUPS'%(r['wavefront_ms'], r['achieved']), 'rescued %d %.2f ms'%(q['pairs'], q['ms']))"
 done
done
