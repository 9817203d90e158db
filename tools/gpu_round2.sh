#!/bin/bash
# Round-2 measurement pass (run under gpurun from the repo root): bench lines, multi-rank lines on one GPU (gloo),
# ncu launch list, full pair-kernel capture, graph-level (in-run, concurrent) profile.  OUT=gpurun_out/<tag>
O=${OUT:-gpurun_out/r02m1}
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
B="timeout 900 python bench.py"
for what in ${WHAT:-bench small large sweep allpairs eps1 multi ll ncu graph}; do
case $what in
 bench) $B --steps 5 > $O/bench_medium.jsonl 2> $O/bench_medium.err ;;
 small) $B --config small > $O/bench_small.jsonl 2> $O/bench_small.err ;;
 large) $B --config large --steps 2 --warmup 3 --no-cpu-baseline > $O/bench_large.jsonl 2> $O/bench_large.err ;;
 sweep) $B --config sweep --steps 1 --warmup 3 > $O/bench_sweep.jsonl 2> $O/bench_sweep.err ;;
 allpairs) $B --mode allpairs --generations 20 --steps 2 --no-cpu-baseline > $O/bench_medium_allpairs_g20.jsonl 2> $O/bench_allpairs.err ;;
 eps1) $B --mode allpairs --dielectric 1 --eps-r 1 --generations 20 --steps 2 > $O/bench_medium_allpairs_eps1_g20.jsonl 2> $O/bench_eps1.err ;;
 multi)
   export VS_BENCH_BACKEND=gloo
   $B --gpus 2 --steps 3 --no-cpu-baseline --no-micro > $O/bench_medium_2rank_queue.jsonl 2> $O/m1.err
   $B --gpus 2 --steps 3 --no-cpu-baseline --no-micro --schedule static --hetero 0:2 > $O/bench_medium_2rank_static_het.jsonl 2> $O/m2.err
   $B --gpus 2 --steps 3 --no-cpu-baseline --no-micro --schedule warmup --hetero 0:2 > $O/bench_medium_2rank_warmup_het.jsonl 2> $O/m3.err
   $B --gpus 2 --steps 3 --no-cpu-baseline --no-micro --schedule queue --chunks-per-rank 4 --slots 2 --hetero 0:2 > $O/bench_medium_2rank_queue_het.jsonl 2> $O/m4.err
   unset VS_BENCH_BACKEND ;;
 ll) VS_GRAPHS=0 timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_medium_g10.csv python tools/prof_run.py --generations 10 > $O/ll.log 2>&1 ;;
 ncu) VS_GRAPHS=0 timeout 900 ncu --set full --clock-control none --import-source on -k regex:cell_pair_kernel -c 2 -f -o $O/pair python tools/prof_run.py --generations 1 > $O/ncu_pair.log 2>&1 ;;
 graph) timeout 900 ncu --graph-profiling graph --profile-from-start off --clock-control none --metrics gpu__time_duration.sum,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_elapsed,smsp__issue_active.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_elapsed,sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_elapsed,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_elapsed,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum,sm__cycles_elapsed.avg.per_second,smsp__average_warps_issue_stalled_wait_per_issue_active.ratio,smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio,smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio,smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio,smsp__average_warps_issue_stalled_no_instruction_per_issue_active.ratio --csv --log-file $O/graph_medium_g10.csv python tools/prof_run.py --generations 10 --graph --replay-only > $O/graph.log 2>&1 ;;
 ref) $B --impl reference > $O/bench_reference.jsonl 2> $O/bench_reference.err ;;
 tests) timeout 1500 python -m pytest tests -x -q -m gpu > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log ;;
 smoke) python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log ;;
esac
done
ls -la $O
