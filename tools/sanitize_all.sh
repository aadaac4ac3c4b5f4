#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over every kernel path
# (tools/sanitize_run.py core + modes) -> gpurun_out/san_<part>_<tool>.txt
for part in core modes; do
  for tool in memcheck racecheck synccheck; do
    timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py $part > gpurun_out/san_${part}_${tool}.txt 2>&1
    echo "$part $tool rc=$? $(tail -1 gpurun_out/san_${part}_${tool}.txt)"
  done
done
