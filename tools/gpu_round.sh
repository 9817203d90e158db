#!/bin/bash
# One GPU measurement pass of the current build (run under gpurun from the repo root):
# GPU tests, bench lines (medium default, small, large), ncu launch list and a full capture of the pair kernel.
set -x
O=${OUT:-gpurun_out/r01s5}
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 1200 python -m pytest tests -x -q -m gpu > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 600 python bench.py > $O/bench_medium.jsonl 2> $O/bench_medium.err
timeout 300 python bench.py --config small > $O/bench_small.jsonl 2> $O/bench_small.err
timeout 600 python bench.py --config large --steps 3 --warmup 3 --no-cpu-baseline > $O/bench_large.jsonl 2> $O/bench_large.err
timeout 900 python bench.py --config sweep --steps 1 --warmup 3 > $O/bench_sweep.jsonl 2> $O/bench_sweep.err
VS_GRAPHS=0 timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_medium_g10.csv python tools/prof_run.py --generations 10 > $O/launches.log 2>&1
VS_GRAPHS=0 timeout 900 ncu --set full --clock-control none --import-source on -k regex:cell_pair_kernel -c 2 -f -o $O/pair python tools/prof_run.py --generations 1 > $O/ncu_pair.log 2>&1
ls -la $O
