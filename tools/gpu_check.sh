#!/bin/bash
# GPU pass of the current build (run under gpurun from the repo root): OUT=gpurun_out/<tag> bash tools/gpu_check.sh [what...]
# what: tests smoke scal bench small large launches ncu
O=${OUT:-gpurun_out/chk}
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
for w in "$@"; do
  case $w in
    smoke) python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log ;;
    tests) timeout 1500 python -m pytest tests -x -q -m gpu > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log ;;
    newtests) timeout 900 python -m pytest tests/test_gpu_shapes.py tests/test_gpu_async.py -x -q > $O/pytest_new.log 2>&1; echo "rc=$?" >> $O/pytest_new.log ;;
    scal) timeout 600 python tools/spot_scaling.py --config medium --spots 500,250,125,63,32,8,1 > $O/scal_medium.json 2>&1 ;;
    scall) timeout 600 python tools/spot_scaling.py --config large --reps 1 > $O/scal_large.json 2>&1 ;;
    scals) timeout 600 python tools/spot_scaling.py --config small --spots 64,32,16,8 > $O/scal_small.json 2>&1 ;;
    bench) timeout 900 python bench.py > $O/bench_medium.jsonl 2> $O/bench_medium.err ;;
    small) timeout 600 python bench.py --config small > $O/bench_small.jsonl 2> $O/bench_small.err ;;
    large) timeout 900 python bench.py --config large --steps 3 --warmup 3 --no-cpu-baseline > $O/bench_large.jsonl 2> $O/bench_large.err ;;
    launches) VS_GRAPHS=0 timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_medium_g10.csv python tools/prof_run.py --generations 10 > $O/launches.log 2>&1 ;;
    ncu) VS_GRAPHS=0 timeout 900 ncu --set full --clock-control none --import-source on -k regex:cell_pair_kernel -c 2 -f -o $O/pair python tools/prof_run.py --generations 1 > $O/ncu_pair.log 2>&1 ;;
  esac
done
ls -la $O
