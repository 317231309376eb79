#!/bin/bash
# compute-sanitizer (memcheck, racecheck, synccheck) over small GPU parity cases
set -u
# build (a no-op when the in-tree library is fresh) outside the sanitizer: nvcc under its injection is not the subject
python -c "from paper_conf_icpp_masw25_b200 import build as B; B.build()" || exit 1
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 \
    python -m pytest tests/test_gpu_parity.py -q -x -k "cfg1_full or chunked or shapes or control_step_sequence or identify or weights" \
    > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool exit=$? $(grep -E 'ERROR SUMMARY|passed|failed' gpurun_out/sanitize_$tool.log | tail -2 | tr '\n' ' ')"
done
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_budget.py -q -x -k "shard_invariance" > gpurun_out/sanitize_budget.log 2>&1
echo "budget memcheck exit=$? $(grep -E 'ERROR SUMMARY|passed|failed' gpurun_out/sanitize_budget.log | tail -2 | tr '\n' ' ')"
# the NEXT rows' kernels (baselines, SLO schedule, move suppression, reference trajectory) and the ABI edges
for f in test_gpu_baselines test_gpu_slo test_gpu_move test_gpu_ref test_gpu_edges; do
  timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python -m pytest tests/$f.py -q -x > gpurun_out/sanitize_$f.log 2>&1
  echo "$f memcheck exit=$? $(grep -E 'ERROR SUMMARY|passed|failed' gpurun_out/sanitize_$f.log | tail -2 | tr '\n' ' ')"
done
