#!/bin/bash
# Round-2 final evidence on one B200 with the final kernels: GPU suite, smoke, the default bench
# line (3 times: repeatability), C3 / C4 / full C5 lines, the reference arm, launch lists,
# device timelines, the small-batch figure, compute-sanitizer.
mkdir -p gpurun_out/final
O=gpurun_out/final
timeout 1200 python -m pytest tests -m gpu -q 2>&1 | tail -3 > $O/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1
for i in 1 2 3; do python bench.py > $O/bench_c2_$i.json 2> $O/bench_c2_$i.err; done
for w in C3 C4; do python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_$w.json 2>/dev/null; done
python bench.py --workload C5 --steps 3 --warmup 3 > $O/bench_c5_full.json 2> $O/bench_c5_full.err
python bench.py --impl reference --steps 2 --warmup 1 > $O/ref.json 2> $O/ref.err
for wl in C2 C3; do
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$wl.csv \
      python bench.py --workload $wl --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline --no-extra > /dev/null 2>&1
  python tools/timeline.py $wl > $O/timeline_$wl.json 2>/dev/null
done
timeout 300 python tools/small_batch.py 1024 > $O/small_batch.json 2> $O/small_batch.err
bash tools/sanitize.sh > $O/sanitize.txt 2>&1
python bench_sw.py > $O/bench_sw.json 2>/dev/null
ls -la $O
