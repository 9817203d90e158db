#!/bin/bash
# compute-sanitizer (memcheck, racecheck, synccheck, initcheck) of tools/sanitize_probe.py; run under gpurun from the repo root
O=${OUT:-gpurun_out/r01s8}; mkdir -p $O; F=$O/compute_sanitizer.txt
echo "# compute-sanitizer on tools/sanitize_probe.py (compacted-copy pair kernel build, HEAD $(cat .git_head 2>/dev/null)): final defaults; VS_GRAPHS=0" > $F
for t in memcheck racecheck synccheck initcheck; do echo "== $t" >> $F; VS_GRAPHS=0 timeout 900 compute-sanitizer --tool $t python tools/sanitize_probe.py 2>&1 | grep -v "^$" | tail -5 >> $F; done
