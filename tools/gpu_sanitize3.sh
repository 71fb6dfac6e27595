#!/bin/bash
mkdir -p gpurun_out/sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 7 python tools/sanitize_cases.py > gpurun_out/sanitizer/${tool}_r02ak.log 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|sanitize cases OK' gpurun_out/sanitizer/${tool}_r02ak.log | tr '\n' ' ')"
done
