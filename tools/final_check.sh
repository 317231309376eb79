#!/bin/bash
# round-end check on one box: compute-sanitizer pass, then the round check (GPU suite, smoke, benches, ncu launch list)
mkdir -p gpurun_out
bash tools/sanitize.sh 2>&1 | tee gpurun_out/sanitize_summary.txt
bash tools/round_check.sh
