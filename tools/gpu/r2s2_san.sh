#!/bin/bash
# compute-sanitizer over tools/sanitize_run.py (round 2, session 2 kernels included)
for tool in memcheck racecheck synccheck initcheck; do
  echo "== compute-sanitizer --tool $tool python tools/sanitize_run.py"
  timeout 1500 compute-sanitizer --tool $tool python tools/sanitize_run.py 2>&1 | tail -3
done
