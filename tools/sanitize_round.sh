#!/bin/bash
# compute-sanitizer (memcheck, racecheck, synccheck, initcheck) of tools/sanitize_probe.py; run under gpurun from the repo root
O=${OUT:-gpurun_out/r02san}; mkdir -p $O; F=$O/compute_sanitizer.txt
echo "# compute-sanitizer on tools/sanitize_probe.py (round-2 build, 4-warp pair-kernel CTAs: list splits 1/2/4, KP 1/2 chunks, coarse item sort, census + launch-interval instrumentation, async entry points); VS_GRAPHS=0" > $F
for t in memcheck racecheck synccheck initcheck; do echo "== $t" >> $F; VS_GRAPHS=0 timeout 1200 compute-sanitizer --tool $t python tools/sanitize_probe.py 2>&1 | grep -v "^$" | tail -5 >> $F; done
cat $F
