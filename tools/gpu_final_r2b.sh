#!/bin/bash
# Round-2 final evidence after the host-path work (pipelined host call, streamed batches): GPU
# suite, smoke, the default bench line 3x, C3 / C4 / full C5 lines, the reference arm, the C2
# launch list, the pipelined-call sweep and the streamed-batch timeline.
mkdir -p gpurun_out/final2
O=gpurun_out/final2
timeout 1200 python -m pytest tests -m gpu -q 2>&1 | tail -3 > $O/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1
for i in 1 2 3; do python bench.py > $O/bench_c2_$i.json 2> $O/bench_c2_$i.err; done
for w in C3 C4; do python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_$w.json 2>/dev/null; done
python bench.py --workload C5 --steps 3 --warmup 3 > $O/bench_c5_full.json 2> $O/bench_c5_full.err
python bench.py --impl reference --steps 2 --warmup 1 > $O/ref.json 2> $O/ref.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C2.csv \
    python bench.py --workload C2 --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline --no-extra > /dev/null 2>&1
bash tools/pipe_sweep.sh > $O/pipe_sweep.txt 2>&1
PIPE_ON=0 bash tools/pipe_sweep.sh >> $O/pipe_sweep.txt 2>&1
python tools/async_timeline.py > $O/async_timeline.txt 2>&1
ls -la $O
