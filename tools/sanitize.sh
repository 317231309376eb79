#!/bin/bash
# compute-sanitizer (memcheck, racecheck, synccheck) over small GPU parity cases
set -u
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 \
    python -m pytest tests/test_gpu_parity.py -q -x -k "cfg1_full or chunked or shapes or control_step_sequence or identify or weights" \
    > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool exit=$? $(grep -E 'ERROR SUMMARY|passed|failed' gpurun_out/sanitize_$tool.log | tail -2 | tr '\n' ' ')"
done
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_budget.py -q -x -k "shard_invariance" > gpurun_out/sanitize_budget.log 2>&1
echo "budget memcheck exit=$? $(grep -E 'ERROR SUMMARY|passed|failed' gpurun_out/sanitize_budget.log | tail -2 | tr '\n' ' ')"
