#!/bin/bash
# compute-sanitizer over tools/sanitize_run.py (run on the GPU box):
#   bash tools/sanitize.sh OUTDIR
set -u
out=${1:-gpurun_out/sanitize}
mkdir -p "$out"
for tool in memcheck racecheck synccheck initcheck; do
  mode=""
  [ "$tool" = "racecheck" ] && mode="quick"
  [ "$tool" = "initcheck" ] && mode="quick"
  extra=""
  [ "$tool" = "synccheck" ] && extra="--num-cuda-barriers 65536"
  timeout 1500 compute-sanitizer --tool $tool $extra --print-limit 50 --error-exitcode 9 \
      --kernel-name kns=3arb python tools/sanitize_run.py $mode > "$out/$tool.log" 2>&1
  echo "$tool rc=$?" | tee -a "$out/summary.txt"
  tail -3 "$out/$tool.log" >> "$out/summary.txt"
done
