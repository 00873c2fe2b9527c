#!/bin/bash
# compute-sanitizer over the small all-kernels workload; one summary line per tool.
# Usage (under gpurun): bash tools/sanitize.sh <tag>
tag=${1:-r02}
out=gpurun_out; mkdir -p $out
python tools/build.py > /dev/null
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 \
      python tools/sanitize_run.py > $out/sanitize_${tool}_$tag.txt 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|sanitize workload ok' $out/sanitize_${tool}_$tag.txt | tr '\n' ' ')"
done
