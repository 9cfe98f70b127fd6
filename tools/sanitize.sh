#!/bin/bash
# compute-sanitizer pass over every kernel family at small ragged shapes (tools/sanitize.py):
# memcheck, racecheck, synccheck.  Logs under gpurun_out/sanitize_<tool>.log; the summary lines
# ("ERROR SUMMARY" / "RACECHECK SUMMARY") are what profiles/<round>_sanitize.md quotes.
# Usage (on the GPU box): bash tools/sanitize.sh [families]
FAM=${1:-hotspot,srad,pathfinder,lud,hotspot3d,dist}
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for fam in ${FAM//,/ }; do
  for tool in memcheck racecheck synccheck; do
    extra=""
    [ "$tool" = memcheck ] && extra="--leak-check no --check-device-heap yes"
    [ "$tool" = racecheck ] && extra="--racecheck-report all"
    echo "=== $tool $fam" >> gpurun_out/sanitize_${tool}.log
    timeout 900 $CS --tool $tool $extra --print-limit 50 --error-exitcode 17 \
      python tools/sanitize.py $fam >> gpurun_out/sanitize_${tool}.log 2>&1
    echo "=== rc=$? $tool $fam" >> gpurun_out/sanitize_${tool}.log
  done
done
grep -h -E "^=== |SUMMARY" gpurun_out/sanitize_*.log > gpurun_out/sanitize_summary.txt
cat gpurun_out/sanitize_summary.txt
