#!/bin/bash
# A/B of FP64 rescue variants: C3 / C4 / C2 rescue time (the FP64 pass incl. its preparation)
# per library, two interleaved repetitions, after a parity check of each variant
for lib in "$@"; do PHMM_LIB=$lib timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "not full_c5" 2>&1 | tail -1 | sed "s|^|$(basename $lib) |"; done
for rep in 1 2; do for wl in C3 C4 C2; do for lib in paper_conf_ipps_wangxc17_b200/libphmm.so "$@"; do
  printf "%-4s %-26s " $wl "$(basename $lib)"
  PHMM_LIB=$lib python bench.py --workload $wl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-extra 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']; q=d['rescue']
print('step %.0f wf %.2f ms rescue %.3f ms (%d pairs)'%(d['value'], r['wavefront_ms'], q['ms'], q['pairs']))"
done; done; done
